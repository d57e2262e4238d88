python -c "import __graft_entry__ as g; g.build()"
for cw in 16 64 256; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=$cw publish=1 reps=1; done
timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=64 publish=0 reps=1
