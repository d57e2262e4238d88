# same-box A/B: the working tree (new) against _ab_old/ (the last commit's package)
# usage: bash tools/gpu_ab_old.sh "<tune args for new and old>"...
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
rm -rf /tmp/abold && mkdir -p /tmp/abold && cp -r tools oracle include /tmp/abold/ && cp -r _ab_old/paper_conf_ipps_nunesc022_b200 /tmp/abold/
(cd /tmp/abold && python -c "from paper_conf_ipps_nunesc022_b200 import build as b; b.build(force=True)" > /dev/null) || exit 1
for a in "$@"; do
  echo "== new: $a"; timeout 600 python tools/tune.py $a | cut -c1-260
  echo "== old: $a"; (cd /tmp/abold && timeout 600 python tools/tune.py $a | cut -c1-260)
done
