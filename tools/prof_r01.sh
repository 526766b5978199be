# Round-1 ncu evidence (run on the GPU box via gpurun from the repo root):
# launch lists of the bench command + ncu --set full of the conv kernels and
# the other kernels, summarised on the box into gpurun_out/prof/ (reports are
# too big to ship); plus the bench lines themselves (not under ncu).
set -x
W=/tmp/prof_raw; rm -rf $W; mkdir -p $W gpurun_out/prof
python __graft_entry__.py >/dev/null
python bench.py > gpurun_out/prof/bench_alexnet.json 2> gpurun_out/prof/bench_alexnet.err
python bench.py --net vgg16 --no-cpu-baseline > gpurun_out/prof/bench_vgg16.json 2> gpurun_out/prof/bench_vgg16.err
for net in alexnet vgg16; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file $W/launches_${net}_bf16.csv python bench.py --net $net --steps 2 --warmup 3 --no-cpu-baseline --no-sweep > $W/launches_${net}.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:conv_tc_kernel -c 13 -o $W/full_${net}_bf16 python bench.py --net $net --steps 1 --warmup 3 --no-cpu-baseline --no-sweep > $W/full_${net}.log 2>&1
done
timeout 600 ncu --set full --clock-control none -k regex:"lrn|stage|softmax|splitk" -c 12 -o $W/full_alexnet_other python bench.py --net alexnet --steps 1 --warmup 3 --no-cpu-baseline --no-sweep > $W/full_other.log 2>&1
python tools/make_profiles.py $W r01 gpurun_out/prof
cp $W/*.log gpurun_out/prof/
ls -la $W gpurun_out/prof
