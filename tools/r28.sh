timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
python -c "import json; d=json.load(open('gpurun_out/bench_default.json')); print('bench', d['value'], d['ms_per_step'], d['roofline']['frac'], 'e2e', d['e2e']['value'], d['e2e']['ms_per_step'])"
timeout 2400 bash tools/launchlist.sh > gpurun_out/launchlist.log 2>&1; echo "launchlist rc=$?"
gzip -f gpurun_out/launches.csv
