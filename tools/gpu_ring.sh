# commit ring A/B: GPU parity, C2 probes (ring vs locked CS, CTA vs cluster)
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
P="timeout 120 python tools/probe.py"
B="C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 ro_adaptive=1"
for a in "server=1 cluster_size=4" "server=0 debug_flags=32"; do
  $P $B $a reps=1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$a', round(d['tx_per_s']/1e6,1), 'M', round(d['abort_rate'],4), {k:v['update'] for k,v in d['aborts'].items()}, d['phase_per_batch'])"
done
timeout 1500 python -m pytest tests/test_gpu_cluster.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
