set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -3
P="timeout 120 python tools/probe.py"
$P C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=2
$P C2 n_tx=16777216 client_warps=448 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=1
$P C4 n_tx=8388608 client_warps=294 publish=1 server_workers=6 ro_streak=8 reps=1
$P C4 n_tx=8388608 client_warps=588 publish=1 server_workers=6 ro_streak=8 reps=1
$P C3 n_tx=4194304 client_warps=64 publish=1 server_workers=6 ro_streak=32 ro_adaptive=1 reps=1
timeout 300 python tools/kv_ways.py --n-tx 4194304 --ways 16,256 2>&1 | tail -3
