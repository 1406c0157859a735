cd $GRAFT_REPO_ROOT
for h in none 64B 128B 256B none; do
  echo "== $h"
  LL_LD_HINT=$h timeout 300 python tools/sweep.py --only big 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l); print(d['case'], d['GBps'], d['frac_6539'])
    except Exception: pass"
done
