cd $GRAFT_REPO_ROOT
python tools/time_model_fit.py > gpurun_out/time_model_fit2.json 2> gpurun_out/tmf2.err
python -c "
import json; d=json.load(open('gpurun_out/time_model_fit2.json')); print(json.dumps(d['fit'])); print(d['compiled_model'])"
