set -x
nproc; free -g | head -2; nvidia-smi; nvidia-smi topo -m | head -20; lscpu | grep -E "Model name|Socket|Core|Thread|NUMA node\(s\)"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/mb tools/alu_microbench.cu && /tmp/mb
