# round-2 final check on one B200: all GPU tests, smoke, default benches (not
# under ncu), then the profile captures of tools/gpu_prof_r02.sh
cd $GRAFT_REPO_ROOT
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/final_gpu_tests.log 2>&1; echo tests=$?; tail -1 gpurun_out/final_gpu_tests.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final_smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/final_smoke.log
timeout 600 python bench.py > gpurun_out/final_bench_alex.json 2> gpurun_out/final_bench_alex.err; echo bench_alex=$?
timeout 600 python bench.py --net vgg16 --no-cpu-baseline > gpurun_out/final_bench_vgg.json 2> gpurun_out/final_bench_vgg.err; echo bench_vgg=$?
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_bench_ref.json 2>&1; echo bench_ref=$?
bash tools/gpu_prof_r02.sh
ls gpurun_out
