python __graft_entry__.py >/dev/null
timeout 1200 python -m pytest tests -m gpu -q -x --timeout 300 -p no:cacheprovider 2>&1 | tail -15
for net in vgg16 alexnet; do timeout 300 python bench.py --net $net --no-cpu-baseline --no-sweep > gpurun_out/bench15_$net.json 2>/dev/null; python -c "import json;d=json.load(open(\"gpurun_out/bench15_$net.json\"));print(d[\"value\"], d[\"roofline\"][\"achieved\"], d[\"roofline\"][\"frac\"], d[\"e2e\"][\"value\"]);[print(l[\"layer\"], l[\"ms\"], l.get(\"tflops\", l.get(\"gbs\")), l.get(\"tile\")) for l in d[\"per_layer\"]]"; done
