python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/gpu_tests_f1.log 2>&1; echo tests=$?; tail -2 gpurun_out/gpu_tests_f1.log
timeout 300 python bench.py > gpurun_out/bench_alex_f1.json 2>gpurun_out/bench_alex_f1.err
timeout 300 python bench.py --net vgg16 --no-cpu-baseline > gpurun_out/bench_vgg_f1.json 2>gpurun_out/bench_vgg_f1.err
for f in gpurun_out/bench_alex_f1.json gpurun_out/bench_vgg_f1.json; do python -c "
import json; d=json.load(open('$f'))
print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e']['value'], d['clocks']['reasons'])
print([(l['layer'], l['ms']) for l in d['per_layer']][-4:])
" || tail -5 $f; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:softmax -c 4 --csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-sweep 2>/dev/null | grep softmax | tail -2
