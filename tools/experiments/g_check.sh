# Full GPU check: build, gpu tests, smoke, default bench (alexnet b256) and vgg16 b64.
mkdir -p gpurun_out/chk
python __graft_entry__.py > gpurun_out/chk/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --timeout 400 -p no:cacheprovider > gpurun_out/chk/pytest.log 2>&1; echo "pytest rc $?"
tail -5 gpurun_out/chk/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/chk/smoke.log 2>&1; echo "smoke rc $?"; tail -2 gpurun_out/chk/smoke.log
nvidia-smi --query-gpu=name,clocks.max.sm,clocks.sm --format=csv > gpurun_out/chk/smi.txt
timeout 600 python bench.py > gpurun_out/chk/bench_alexnet.json 2> gpurun_out/chk/bench_alexnet.err; echo "bench alexnet rc $?"
timeout 600 python bench.py --net vgg16 --no-cpu-baseline > gpurun_out/chk/bench_vgg16.json 2> gpurun_out/chk/bench_vgg16.err; echo "bench vgg rc $?"
timeout 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/chk/bench_ref.json 2>&1; echo "ref rc $?"
cat MEASURED_PEAKS.json > gpurun_out/chk/peaks.json 2>/dev/null
