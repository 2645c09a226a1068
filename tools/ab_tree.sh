#!/bin/bash
# Same-box A/B of a source change: tools/ab_patch.diff is the change (applied in this tree);
# the baseline tree is a copy with the patch reversed, built on the box.  Args: reps [lg]
cd "$GRAFT_REPO_ROOT"; R=${1:-3}; LG=${2:-27}
rm -rf /tmp/alt && cp -r . /tmp/alt && (cd /tmp/alt && patch -s -R -p1 < tools/ab_patch.diff && python -c "import __graft_entry__ as g; g.build()") || { echo "baseline build failed"; exit 1; }
for i in $(seq $R); do
  (cd "$GRAFT_REPO_ROOT" && timeout 200 python tools/${AB:-ab_del.py} ${ABARGS:-0 $LG 1} | head -1 | sed "s/^/new: /")
  (cd /tmp/alt && timeout 200 python tools/${AB:-ab_del.py} ${ABARGS:-0 $LG 1} | head -1 | sed "s/^/old: /")
done
