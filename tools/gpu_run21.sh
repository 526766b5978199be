cd $GRAFT_REPO_ROOT
timeout -s KILL 900 python tools/tune_demo.py 64 > gpurun_out/tune_demo_r02.json 2> gpurun_out/tune_demo.err; echo "tune rc=$?"
timeout -s KILL 1200 python tools/config3.py > gpurun_out/config3_r02.json 2> gpurun_out/config3.err; echo "config3 rc=$?"
timeout -s KILL 300 python tools/released_sms_demo.py > gpurun_out/released_sms_r02.json 2>&1; echo "rsd rc=$?"
