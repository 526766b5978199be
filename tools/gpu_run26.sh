cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python tools/tune_demo.py 256 > gpurun_out/tune_demo_r02_b256.json 2> gpurun_out/tune_demo.err; echo "tune rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/tune_demo_r02_b256.json'))
print([ (p['layer'], round(p['time'],4), round(p['entropy'],4)) for p in d['path']]); print(d['calibration'])"
