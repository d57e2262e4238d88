set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python tools/sweep_c5.py --check --out gpurun_out/c5_sweep.jsonl > gpurun_out/c5.log 2>&1; tail -2 gpurun_out/c5.log
timeout 900 python tools/ablation.py --check --warps 56 --out gpurun_out/ablation_w56.jsonl 2>&1 | tail -1
timeout 900 python tools/ablation.py --check --out gpurun_out/ablation_full.jsonl 2>&1 | tail -1
timeout 900 python tools/kv_ways.py --check --n-tx 4194304 --out gpurun_out/kv_ways.jsonl 2>&1 | tail -1
