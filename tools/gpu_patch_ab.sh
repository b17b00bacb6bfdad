#!/bin/bash
# Same-box A/B of a source patch: bench A (tree as shipped) and B (tree + PATCH),
# interleaved A B A B so box drift cancels.  usage: tools/gpu_patch_ab.sh TAG PATCH [bench args]
TAG=$1; PATCH=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
build() { python -c "from paper_conf_ipps_yuphs21_b200 import build as b; b.build(force=True)" > $OUT/build_$1.log 2>&1 || { echo "build $1 failed"; tail -5 $OUT/build_$1.log; exit 1; }; cp paper_conf_ipps_yuphs21_b200/libarbalest.so /tmp/lib_$1.so; }
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
build A
patch -p1 < $PATCH > $OUT/patch.log || { echo "patch failed"; cat $OUT/patch.log; exit 1; }
build B
if [ -n "$PYTEST_B" ]; then timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_B.log 2>&1; echo "pytest B rc=$?"; tail -2 $OUT/pytest_B.log; fi
if [ -n "$NCU_KERNEL" ]; then   # per-launch kernel durations under ncu (serialised, cold): less noisy than the bench
  for v in A B; do
    cp /tmp/lib_$v.so paper_conf_ipps_yuphs21_b200/libarbalest.so
    timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"$NCU_KERNEL" --csv \
      python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu "$@" > $OUT/ncu_$v.csv 2> $OUT/ncu_$v.err
    python - $OUT/ncu_$v.csv $v <<'PY'
import csv, io, sys
t = open(sys.argv[1]).read(); t = t[t.find('"ID"'):]
ms = [float(r["Metric Value"].replace(",", "")) / (1e6 if r["Metric Unit"] == "ns" else 1e3 if r["Metric Unit"] == "us" else 1)
      for r in csv.DictReader(io.StringIO(t)) if r.get("Metric Name") == "gpu__time_duration.sum"]
print(sys.argv[2], "ncu ms per launch:", [round(x, 4) for x in ms], "sum", round(sum(ms), 4))
PY
  done
fi
for v in A B A B; do
  cp /tmp/lib_$v.so paper_conf_ipps_yuphs21_b200/libarbalest.so
  timeout 300 python bench.py --no-e2e --no-cpu "$@" > $OUT/bench_$v.json 2> $OUT/bench_$v.err
  python -c "import json;d=json.load(open('$OUT/bench_$v.json'));print('$v',round(d['ms_per_step'],3),{k:round(v,3) for k,v in d['roofline']['phase_ms_per_step'].items() if 'in control' not in k})"
done
