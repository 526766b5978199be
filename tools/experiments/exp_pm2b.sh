python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_perforation.py -x -q 2>&1 | tail -3
timeout 200 python tools/variant_layers.py 256 2>&1 | grep -v plan
