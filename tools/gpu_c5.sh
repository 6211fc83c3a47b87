exec > gpurun_out/c5.log 2>&1
for kt in u64 f32; do
timeout 900 python bench.py --key-type $kt --keys 2e9 --steps 5 --warmup 3 --het --cpu-seconds 5 > gpurun_out/c5_$kt.json 2> gpurun_out/c5_$kt.err
echo "$kt rc=$?"; tail -c 200 gpurun_out/c5_$kt.err
python -c "import json; d=json.load(open('gpurun_out/c5_$kt.json')); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['het_baseline']['value'])"
done
