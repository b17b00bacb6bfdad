TAG=${TAG:-side}; mkdir -p gpurun_out/$TAG
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q -k "runs_fuzz or config2 or fuzz_small or fuzz_large or big or flush_cuts or split_parts or hot_word" > gpurun_out/$TAG/pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/$TAG/pytest.log; tail -2 gpurun_out/$TAG/pytest.log
timeout 600 python bench.py --no-e2e --no-cpu --steps 3 > gpurun_out/$TAG/bench.json 2> gpurun_out/$TAG/bench.err
python -c "
import json;d=json.load(open('gpurun_out/$TAG/bench.json'));c=d['config']
print(round(d['ms_per_step'],2),{k:round(v,2) for k,v in d['roofline']['phase_ms_per_step'].items()},c['segments_rank0'],c['chunks_all_fast_run_rank0'])
for k,v in d['workloads'].items(): print(k, round(v['ms_per_step'],2), round(v['path_frac'],3), {kk:round(x,2) for kk,x in v['phase_ms_per_step'].items()})"
