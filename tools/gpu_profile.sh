# Round-end evidence: bench lines (both arms), the ncu launch list of the
# bench command, and one full ncu capture of the fused kernel at the bench
# workload.  Outputs under gpurun_out/ (copied into profiles/ by hand).
set -x
TAG=${TAG:-r01}
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -1 gpurun_out/bench_$TAG.json
timeout 600 python bench.py --impl reference > gpurun_out/bench_ref_$TAG.json 2>&1; tail -1 gpurun_out/bench_ref_$TAG.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu_$TAG.log 2>&1
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:csmv_fused -s 3 -c 1 \
  -o gpurun_out/prof_fused_$TAG python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/prof_fused_$TAG.log 2>&1
tail -3 gpurun_out/prof_fused_$TAG.log
