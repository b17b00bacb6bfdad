#!/bin/bash
# Iteration round trip: build, a pytest selection (PYK), a short bench (first 2 batches),
# optionally (NCU=1) an ncu --set full capture of k_partition / k_replay on one batch.
# usage: tools/gpu_iter.sh TAG
TAG=${1:-iter}; OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1 || { tail $OUT/build.log; exit 1; }
timeout ${PYT:-900} python -m pytest tests -m gpu -x -q ${PYK:+-k "$PYK"} > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
tail -n 3 $OUT/pytest.log
timeout 300 python bench.py --no-e2e --no-cpu --no-side --max-batches ${MB:-2} --steps 2 > $OUT/bench.json 2> $OUT/bench.err
python -c "import json;d=json.load(open('$OUT/bench.json'));c=d['config'];print(round(d['ms_per_step'],3),{k:round(v,3) for k,v in d['roofline']['phase_ms_per_step'].items()},c['replay_steps_fast_sort_run_rank0'],c['segments_rank0'],c['chunks_all_fast_run_rank0'])" || tail $OUT/bench.err
if [ -n "$NCU" ]; then
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_partition|k_replay" -c 2 -o $OUT/full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-side --max-batches 1 > $OUT/ncu_full.log 2>&1
  tail -n 1 $OUT/ncu_full.log
fi
