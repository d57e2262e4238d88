set -x
python -c "import __graft_entry__ as g; g.build()"
P="timeout 120 python tools/probe.py"
$P C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=3
