#!/bin/bash
# Quick GPU round trip: build, GPU parity tests, bench without e2e/cpu legs.
TAG=${1:-quick}; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q "$@" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
timeout 300 python bench.py --no-e2e --no-cpu > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
for f in smoke.log pytest.log bench.err; do tail -n 3 $OUT/$f; done
python -c "import json;d=json.load(open('$OUT/bench.json'));print(d['ms_per_step'],d['value'],d['roofline']['phase_ms_per_step'])"
if [ -n "$NCU" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"$NCU" -c 2 -o $OUT/full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > $OUT/ncu_full.log 2>&1
  tail -n 2 $OUT/ncu_full.log
fi
if [ -n "$LAUNCHES" ]; then
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > $OUT/ncu_launch.log 2>&1
fi
