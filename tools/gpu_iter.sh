# iteration check: targeted GPU tests + bench (sweep) + optional extra command
cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest ${TESTS:-tests} -m gpu -q -x -p no:cacheprovider > gpurun_out/it_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/it_tests.log
timeout 600 python bench.py --no-extra --no-cpu-baseline > gpurun_out/it_bench.json 2> gpurun_out/it_bench.err; echo bench=$?
python - <<'P'
import json
d=json.load(open('gpurun_out/it_bench.json'))
print('B=256', d['value'], d['ms_per_step'], d['roofline']['frac'])
for l in d['per_layer']: print('  ', l['layer'], l['ms'], l.get('roofline_frac'))
for b,v in d['sweep'].items(): print(b, v['ms'], v['img_s'], {k: round(x[0]*1000,1) for k,x in v['layers'].items()})
P
if [ -n "$EXTRA" ]; then bash -c "$EXTRA"; fi
