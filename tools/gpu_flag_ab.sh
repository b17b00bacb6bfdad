#!/bin/bash
# Same-box A/B/C of compile-time variants: tools/gpu_flag_ab.sh TAG "FLAGS_A" "FLAGS_B" ["FLAGS_C"] -- [bench args]
# Each variant is built with ARB_NVCC_FLAGS=<flags>; benches run interleaved (A B C A B C).
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
V=(); while [ $# -gt 0 ] && [ "$1" != "--" ]; do V+=("$1"); shift; done; shift
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for i in "${!V[@]}"; do
  ARB_NVCC_FLAGS="${V[$i]}" python -c "from paper_conf_ipps_yuphs21_b200 import build as b; b.build(force=True)" > $OUT/build_$i.log 2>&1 || { echo "build $i failed"; tail -3 $OUT/build_$i.log; exit 1; }
  cp paper_conf_ipps_yuphs21_b200/libarbalest.so /tmp/lib_$i.so
done
for r in 1 2; do for i in "${!V[@]}"; do
  cp /tmp/lib_$i.so paper_conf_ipps_yuphs21_b200/libarbalest.so
  timeout 300 python bench.py --no-e2e --no-cpu "$@" > $OUT/bench_${i}_$r.json 2> $OUT/bench_${i}_$r.err
  python -c "import json;d=json.load(open('$OUT/bench_${i}_$r.json'));print('[${V[$i]}]',round(d['ms_per_step'],3),{k:round(v,3) for k,v in d['roofline']['phase_ms_per_step'].items() if 'in control' not in k})"
done; done
