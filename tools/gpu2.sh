set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
for cw in 32 64 128 256; do for pub in 0 1; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=$cw publish=$pub reps=1; done; done
timeout 120 python tools/probe.py C3 n_tx=4194304 client_warps=128 publish=1 reps=1
timeout 120 python tools/probe.py C3 n_tx=4194304 client_warps=0 publish=1 reps=1
timeout 120 python tools/probe.py C1 publish=1 reps=1
