#!/bin/bash
# Same-box A/B of runtime switches: tools/gpu_env_ab.sh TAG "ENV_A" "ENV_B" ... -- [bench args]
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
V=(); while [ $# -gt 0 ] && [ "$1" != "--" ]; do V+=("$1"); shift; done; shift
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do for i in "${!V[@]}"; do
  env ${V[$i]} timeout 300 python bench.py --no-e2e --no-cpu "$@" > $OUT/bench_${i}_$r.json 2> $OUT/bench_${i}_$r.err
  python -c "import json;d=json.load(open('$OUT/bench_${i}_$r.json'));c=d['config'];print('[${V[$i]}]',round(d['ms_per_step'],3),{k:round(v,3) for k,v in d['roofline']['phase_ms_per_step'].items() if 'in control' not in k}, c['replay_steps_fast_sort_run_rank0'])"
done; done
