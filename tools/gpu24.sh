set -x
python -c "import __graft_entry__ as g; g.build()"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/cs_ubench tools/ubench/cs_ubench.cu && timeout 60 /tmp/cs_ubench
timeout 1200 python -m pytest tests/test_gpu_ablation.py tests/test_gpu_kv.py -x -q 2>&1 | tail -15
timeout 900 python tools/ablation.py --check --out gpurun_out/ablation.jsonl 2>&1 | tail -30
timeout 1200 python tools/kv_ways.py --check --n-tx 2097152 --out gpurun_out/kv_ways.jsonl 2>&1 | tail -10
