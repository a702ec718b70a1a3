#!/bin/bash
# A/B of library build variants on the bench's headline line (dev helper, run under gpurun):
#   tools/ab_bench.sh "<bench args>" tagA tagB ...   (tag "base" = _lib/librrl.so)
# Variants run interleaved, twice; prints tag, step ms, updatePartials ms, roofline frac, reroot speedup.
ARGS="$1"; shift
L=paper_conf_ipps_ayresc18_b200/_lib
for rep in 1 2; do
  for t in "$@"; do
    if [ "$t" = base ]; then P=$L/librrl.so; else P=$L/librrl-$t.so; fi
    RRL_LIB_PATH=$P timeout 600 python bench.py $ARGS 2>/dev/null | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read())
r=d.get('reroot',{})
print('$t', 'rep $rep', 'step %.4f ms' % d['ms_per_step'], 'up %.4f ms' % d['updatePartials']['ms_per_pass'],
      'frac %.3f' % d['roofline']['frac'], 'reroot %.3f' % r.get('updatePartials_speedup', 0), 'orig_up %.4f' % r.get('original_updatePartials_ms', 0))"
  done
done
