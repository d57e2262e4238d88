python -c "import __graft_entry__ as g; g.build()"
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 2>&1 | tail -1
# launch list of the bench command (cold-cache, serialised)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
# full capture of the fused kernel on the bench workload (reduced n_tx)
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:csmv_fused -s 1 -c 1 -o gpurun_out/prof_bench_r01 python bench.py --steps 1 --warmup 1 --no-cpu-baseline --n-tx 2097152 > gpurun_out/prof_bench.log 2>&1
tail -2 gpurun_out/prof_bench.log
