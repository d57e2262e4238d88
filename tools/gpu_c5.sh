# C5 sweep (150 points, oracle parity on each) + round-end profiles of the C2 bench
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 3000 python tools/sweep_c5.py --check --out gpurun_out/c5_sweep.jsonl > gpurun_out/c5_sweep.log 2>&1; tail -2 gpurun_out/c5_sweep.log
TAG=r01c bash tools/gpu_profile.sh
