#!/bin/bash
# A/B round trip: GPU parity tests, then the bench for each extra-argument set.
# usage: tools/gpu_ab.sh TAG "ARGS_A" "ARGS_B" ...   (PYTEST=0 skips the tests)
TAG=${1:-ab}; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
tail -n 2 $OUT/smoke.log
if [ "${PYTEST:-1}" != 0 ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
  tail -n 3 $OUT/pytest.log
fi
i=0
for a in "$@"; do
  timeout 300 python bench.py --no-e2e --no-cpu $a > $OUT/bench$i.json 2> $OUT/bench$i.err
  echo "[$a] rc=$?"; python -c "import json;d=json.load(open('$OUT/bench$i.json'));print(d['ms_per_step'],d['value'],{k:round(v,3) for k,v in d['roofline']['phase_ms_per_step'].items()})"
  i=$((i+1))
done
