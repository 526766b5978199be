cd $GRAFT_REPO_ROOT
timeout 600 python bench.py > gpurun_out/bench_g.json 2> gpurun_out/bench_g.err
echo "bench rc=$?"
python tools/time_model_fit.py > gpurun_out/time_model_fit.json 2> gpurun_out/tmf.err
python tools/released_sms_demo.py > gpurun_out/released_sms.json 2> gpurun_out/rsd.err
ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_b256_g.csv python bench.py --minimal --steps 20 --warmup 5 > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none -s 80 -c 320 --csv --log-file gpurun_out/launches_b1_g.csv python bench.py --minimal --steps 20 --warmup 5 --batch 1 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:"lrn_bulk" -s 2 -c 2 -o gpurun_out/lrn_bulk_prof python bench.py --minimal --steps 2 --warmup 3 > /dev/null 2>&1
echo done
