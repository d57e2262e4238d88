python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
B="C2 n_tx=16777216 publish=1 server_workers=6 server_combine=4 ro_streak=8 ro_adaptive=1 log_mode=0"
for cw in 294 441 588 882 1176; do timeout 120 python tools/phases.py $B client_warps=$cw | cut -c 150-700; done
for rs in 4 16; do timeout 120 python tools/phases.py $B client_warps=588 ro_streak=$rs | cut -c 150-700; done
