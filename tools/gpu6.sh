python -c "import __graft_entry__ as g; g.build()"
for sw in 1 2 4 8 14; do timeout 120 python tools/probe.py C2 n_tx=2097152 client_warps=64 publish=1 server_workers=$sw reps=1; done
timeout 120 python tools/probe.py C2 n_tx=2097152 client_warps=16 publish=1 server_workers=4 reps=1
timeout 120 python tools/probe.py C2 n_tx=2097152 client_warps=128 publish=1 server_workers=4 reps=1
timeout 120 python tools/probe.py C2 n_tx=2097152 client_warps=64 publish=0 server_workers=4 reps=1
timeout 300 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
