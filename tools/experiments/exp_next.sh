python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests_next.log 2>&1; echo tests=$?; tail -3 gpurun_out/gpu_tests_next.log
timeout 900 python tools/config3.py > gpurun_out/config3.json 2> gpurun_out/config3.err; echo config3=$?; tail -3 gpurun_out/config3.err
