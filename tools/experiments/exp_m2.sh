python __graft_entry__.py > gpurun_out/build.log 2>&1 || { tail gpurun_out/build.log; exit 1; }
timeout 120 python -m pytest tests/test_gpu_padded.py -x -q -k two_subtiles 2>&1 | tail -3
timeout 300 python -m pytest tests/test_gpu_padded.py tests/test_gpu_parity.py -x -q 2>&1 | tail -3
for L in vgg1_2+pm vgg2_2+pm conv1p+pm conv2p+pm vgg3_2+pm; do
  for MS in 1 2; do echo "== $L msub=$MS"; PCNN_PM_MSUB=$MS timeout 60 python tools/one_layer.py $L 64 20; done
done
for L in conv1p+pm conv2p+pm; do echo "== $L B256 auto"; timeout 60 python tools/one_layer.py $L 256 20; done
timeout 300 python bench.py --no-sweep --no-cpu-baseline > gpurun_out/bench_alex3.json 2>&1
timeout 300 python bench.py --net vgg16 --no-sweep --no-cpu-baseline > gpurun_out/bench_vgg3.json 2>&1
for f in gpurun_out/bench_alex3.json gpurun_out/bench_vgg3.json; do python -c "
import json; d=json.load(open('$f'))
print(d['value'], d['ms_per_step'], d['roofline']['frac'])
for l in d['per_layer']: print(l)
" || tail -5 $f; done
