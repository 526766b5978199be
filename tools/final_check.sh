# final round check: build, all GPU tests, smoke, default benches (not under ncu)
python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/final_gpu_tests.log 2>&1; echo tests=$?; tail -1 gpurun_out/final_gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 300 python bench.py > gpurun_out/final_bench_alex.json 2> gpurun_out/final_bench_alex.err
timeout 300 python bench.py --net vgg16 --no-cpu-baseline > gpurun_out/final_bench_vgg.json 2> gpurun_out/final_bench_vgg.err
timeout 200 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_bench_ref.json 2>&1
for f in gpurun_out/final_bench_alex.json gpurun_out/final_bench_vgg.json; do python -c "
import json; d=json.load(open('$f'))
print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e']['value'], d['gpu_launches'], d['clocks'])
"; done
cut -c1-200 gpurun_out/final_bench_ref.json
