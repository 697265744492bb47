#!/bin/bash
# Same-box A/B of the working tree against a committed revision (box-to-box variance of
# the products step is ~1-2 %, larger than most scheduling changes).
#   here:      bash tools/ab_rev.sh prepare [REV]   # builds REV (default HEAD) into .abrev/
#   under gpurun: bash tools/ab_rev.sh run [ENV...] # alternates the two trees, 3 reps each
set -u
ROOT=$(cd "$(dirname "$0")/.." && pwd)
if [ "${1:-}" = prepare ]; then
  rev=${2:-HEAD}
  rm -rf "$ROOT/.abrev" && mkdir -p "$ROOT/.abrev"
  git -C "$ROOT" archive "$rev" | tar -x -C "$ROOT/.abrev"
  (cd "$ROOT/.abrev" && python -c "import __graft_entry__ as g; g.build()") && echo "built $rev in .abrev"
  exit $?
fi
shift
mkdir -p "$ROOT/gpurun_out"
for rep in 1 2 3; do
  a=$(cd "$ROOT/.abrev" && env "$@" timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 60 --warmup 10 2>/dev/null | tail -1 | python -c "import json,sys; print(round(json.loads(sys.stdin.read())['ms_per_step'],4))")
  b=$(cd "$ROOT" && env "$@" timeout 300 python bench.py --no-planner --no-cpu-baseline --steps 60 --warmup 10 2>/dev/null | tail -1 | python -c "import json,sys; print(round(json.loads(sys.stdin.read())['ms_per_step'],4))")
  echo "rep $rep  rev $a  tree $b"
done
