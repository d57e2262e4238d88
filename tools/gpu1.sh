set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" 
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -20
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -30
for cw in 64 256 1024 0; do for pub in 0 1; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=$cw publish=$pub reps=2; done; done
