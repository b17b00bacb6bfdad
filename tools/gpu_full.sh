#!/bin/bash
# Full round trip: build + smoke, default bench line (with e2e, cpu_baseline, side configs),
# launch list of one step, the whole-trace parity tests.  usage: tools/gpu_full.sh TAG
TAG=${1:-full}; OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/smi.txt 2>&1
nproc > $OUT/nproc.txt; free -g >> $OUT/nproc.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-side > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_partition|k_replay" -c 2 -o $OUT/full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu --no-side --max-batches 1 > $OUT/ncu_full.log 2>&1
timeout ${PYT:-1800} python -m pytest tests -m gpu -x -q ${PYK:+-k "$PYK"} > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
tail -n 2 $OUT/smoke.log $OUT/bench.err $OUT/pytest.log
