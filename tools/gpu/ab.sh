#!/bin/bash
# Same-box A/B of bench.py option sets, alternating over R rounds (how every "measured X vs Y"
# in DESIGN.md was taken; one-off runner scripts of earlier sessions were folded into this):
#   tools/gpu/ab.sh TAG CONFIG STEPS R "setA" "setB" ...
# a set is a space-separated list of Solver.OPTIONS key=value pairs ("-" = defaults), e.g.
#   tools/gpu/ab.sh serp C2 10 2 "serp=0" "serp=1"
# lines land in gpurun_out/ab_TAG_<round>_<set>.json
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
TAG=$1; CFG=$2; STEPS=$3; R=$4; shift 4
for rep in $(seq 1 $R); do
  for set in "$@"; do
    opts=""
    if [ "$set" != "-" ]; then for kv in $set; do opts="$opts --opt $kv"; done; fi
    name=$(echo "$set" | tr ' =' '_-')
    timeout 1200 python bench.py --config $CFG --no-cpu --no-gmres --steps $STEPS $opts \
      > gpurun_out/ab_${TAG}_${rep}_${name}.json 2>> gpurun_out/ab_${TAG}.err
  done
done
