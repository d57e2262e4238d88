set -x
P="timeout 120 python tools/probe.py"
for v in v1 v2 e427 v1 v2; do
  cp tools/alt_server_$v.cuh paper_conf_ipps_nunesc022_b200/csrc/server.cuh
  python -c "from paper_conf_ipps_nunesc022_b200 import build; build.build(force=True)"
  echo "== $v"
  $P C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=2 | cut -c1-120
done
