python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests_f2.log 2>&1; echo tests=$?; tail -2 gpurun_out/gpu_tests_f2.log
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 300 python bench.py > gpurun_out/bench_alex_f2.json 2>gpurun_out/bench_alex_f2.err
timeout 300 python bench.py --net vgg16 --no-cpu-baseline > gpurun_out/bench_vgg_f2.json 2>gpurun_out/bench_vgg_f2.err
for f in gpurun_out/bench_alex_f2.json gpurun_out/bench_vgg_f2.json; do python -c "
import json; d=json.load(open('$f'))
print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e'], d['clocks']['reasons'])
" || tail -5 $f; done
timeout 120 python bench.py --impl reference --steps 2 --warmup 1 | cut -c1-300
