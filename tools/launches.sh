# per-kernel launch list (ncu gpu__time_duration, cold, serialised) of the bench step
python __graft_entry__.py > /dev/null 2>&1 || exit 1
mkdir -p gpurun_out/prof
for net in alexnet vgg16; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/prof/launches_${net}_bf16.csv python bench.py --net $net --steps 2 --warmup 3 --no-cpu-baseline --no-sweep > /dev/null 2>&1
done
