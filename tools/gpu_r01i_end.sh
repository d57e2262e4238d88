set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_r01i.log 2>&1; tail -2 gpurun_out/pytest_gpu_r01i.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
TAG=r01i bash tools/gpu_profile.sh
for W in C3 C4; do timeout 600 python bench.py --config $W --no-cpu-baseline > gpurun_out/bench_${W}_r01i.json 2>/dev/null; tail -1 gpurun_out/bench_${W}_r01i.json | cut -c1-200; done
