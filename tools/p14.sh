mkdir -p gpurun_out
TAG=${1:-p14}
timeout 300 python -m pytest tests/test_gpu_f16.py -x -q > gpurun_out/${TAG}_f16.txt 2>&1
timeout 600 python -m pytest tests -m gpu -q > gpurun_out/${TAG}_pytest.txt 2>&1
timeout 900 python tools/bench_configs.py c1 c3 c2 sweep f16 > gpurun_out/${TAG}_configs.jsonl 2> gpurun_out/${TAG}_configs.err
HOST_REFS=1000000 timeout 900 python tools/bench_configs.py host >> gpurun_out/${TAG}_configs.jsonl 2>> gpurun_out/${TAG}_configs.err
