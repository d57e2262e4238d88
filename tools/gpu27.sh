set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 60 python -m pytest tests/test_gpu_kv.py tests/test_gpu_parity.py -q -x 2>&1 | tail -2
P="timeout 120 python tools/probe.py"
$P C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=1
$P C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=16 ro_adaptive=1 reps=1
$P C4 n_tx=8388608 client_warps=294 publish=1 server_workers=6 ro_streak=8 reps=1
$P C4 n_tx=8388608 client_warps=294 publish=1 server_workers=6 ro_streak=32 ro_adaptive=1 reps=1
$P C4 n_tx=8388608 client_warps=294 publish=1 server_workers=6 ro_streak=8 debug_flags=16 reps=1
timeout 300 python tools/kv_ways.py --n-tx 4194304 --ways 16,256 2>&1 | tail -3
