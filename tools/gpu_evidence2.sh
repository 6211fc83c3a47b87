exec > gpurun_out/evidence2.log 2>&1
nvidia-smi --query-gpu=name,clocks.max.sm --format=csv,noheader
timeout 900 python bench.py > gpurun_out/bench_e2.json 2> gpurun_out/bench_e2.err
tail -c 200 gpurun_out/bench_e2.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_e2.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1
echo "ncu list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:onesweep -s 6 -c 1 -o /tmp/os_e2 python tools/prof_radix.py 4e9 u32 2 > /dev/null 2>&1
echo "ncu full rc=$?"
python tools/ncu_summary.py /tmp/os_e2.ncu-rep 20 > gpurun_out/os_e2_ncu.txt 2>&1
ncu -i /tmp/os_e2.ncu-rep --page raw --csv 2>/dev/null | python3 -c "
import csv,sys,json
r=list(csv.reader(sys.stdin)); h,u,v=r[0],r[1],r[2]
d=dict(zip(h,v)); uu=dict(zip(h,u))
def gb(k):
    x=float(d[k].replace(',',''))
    return x*{'Gbyte':1e9,'Mbyte':1e6,'Kbyte':1e3,'byte':1}[uu[k]]
rd, wr = gb('dram__bytes_read.sum'), gb('dram__bytes_write.sum')
json.dump({'source':'ncu --set full --clock-control none, onesweep pass 3 of 4 (tools/prof_radix.py 4e9 u32 2), round-1 final kernel (profiles/r1_onesweep_4e9_ncu.txt)','keys_per_launch':4000000000,'dram_bytes_read':rd,'dram_bytes_write':wr,'dram_bytes_per_launch':rd+wr,'algorithmic_bytes_per_launch':32e9}, open('gpurun_out/onesweep_traffic_e2.json','w'), indent=1)
"
cat gpurun_out/bench_e2.json | head -c 600
