mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/p7_pytest.txt 2>&1
bash tools/ab.sh p7 base fake
timeout 300 python bench.py > gpurun_out/p7_bench.json 2> gpurun_out/p7_bench.err
