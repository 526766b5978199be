cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout -s KILL 600 compute-sanitizer --tool $tool --print-limit 20 python -m pytest -q -p no:cacheprovider \
    "tests/test_gpu_parity.py::test_cifar_quick_config0" \
    "tests/test_gpu_fc.py::test_fc_kernel_parity" \
    "tests/test_gpu_parity.py::test_lrn_pool_kernel_shapes" > gpurun_out/sanitizer/$tool.log 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitizer/$tool.log
done
timeout -s KILL 600 python -m pytest tests/test_gpu_time_model.py tests/test_gpu_tuning.py -q -p no:cacheprovider 2>&1 | tail -3
timeout -s KILL 600 python tools/time_model_fit.py > gpurun_out/time_model_fit3.json 2>&1
python -c "import json; d=json.load(open('gpurun_out/time_model_fit3.json')); print(json.dumps(d['fit'])); print(d['compiled_model'])"
