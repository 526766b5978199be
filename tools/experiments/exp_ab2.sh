python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_padded.py -x -q 2>&1 | tail -2
for spec in "conv2p+pm 256" "conv4+pm 256" "conv5+pm 256" "vgg1_2+pm 64" "vgg2_2+pm 64"; do
  set -- $spec
  echo "== $1 B=$2 head: $(PCNN_LIB=build/ab/libpcnn_head.so timeout 60 python tools/one_layer.py $1 $2 30 | tail -1)"
  echo "== $1 B=$2 new : $(timeout 60 python tools/one_layer.py $1 $2 30 | tail -1)"
done
timeout 300 python bench.py --no-sweep --no-cpu-baseline > gpurun_out/bench_alex4.json 2>&1
timeout 300 python bench.py --net vgg16 --no-sweep --no-cpu-baseline > gpurun_out/bench_vgg4.json 2>&1
for f in gpurun_out/bench_alex4.json gpurun_out/bench_vgg4.json; do python -c "
import json; d=json.load(open('$f'))
print(d['value'], d['ms_per_step'], d['roofline']['frac'], d['e2e']['value'])
print([(l['layer'], l['ms']) for l in d['per_layer']])
" || tail -5 $f; done
