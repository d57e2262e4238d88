set -x
python -c "import __graft_entry__ as g; g.build()"
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/cs_ubench tools/ubench/cs_ubench.cu && timeout 60 /tmp/cs_ubench
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
P="timeout 120 python tools/probe.py"
$P C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=2
$P C4 n_tx=8388608 client_warps=294 publish=1 server_workers=6 ro_streak=8 reps=1
timeout 300 python bench.py --steps 5 --no-cpu-baseline | tail -1
