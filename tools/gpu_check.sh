#!/bin/bash
# One GPU round trip: build, GPU parity tests, bench, launch list, ncu capture of the hot kernels.
# usage: tools/gpu_check.sh TAG [pytest-args...]
set -x
TAG=${1:-run}; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > $OUT/smi.txt 2>&1
nproc > $OUT/nproc.txt; free -g >> $OUT/nproc.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q "$@" > $OUT/pytest.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest.log
timeout 600 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > $OUT/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_partition|k_replay" -c 2 -o $OUT/full python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu > $OUT/ncu_full.log 2>&1
ls -la $OUT
