# per-kernel durations (ncu launch list) for one bench step; args: env settings
python __graft_entry__.py > /dev/null 2>&1
mkdir -p gpurun_out/launch
for v in "" "$@"; do for net in alexnet vgg16; do
  tag=$(echo "$net$v" | tr '=' '_')
  env $v timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launch/$tag.csv python bench.py --net $net --steps 1 --warmup 3 --no-sweep --no-cpu-baseline > /dev/null 2>&1
  python tools/launch_summary.py gpurun_out/launch/$tag.csv "$tag"
done; done
