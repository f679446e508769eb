timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/road_launch.csv python scripts/profile_run.py --config road_50m_110m --runs 1 > gpurun_out/road_launch.log 2>&1
python scripts/launch_table.py gpurun_out/road_launch.csv | head -30
python - <<'PY'
import csv, collections
rows=[r for r in csv.reader(open('gpurun_out/road_launch.csv')) if r]
hi=next(i for i,r in enumerate(rows) if "Kernel Name" in r); h=rows[hi]
ik,im,iv,iid=h.index("Kernel Name"),h.index("Metric Name"),h.index("Metric Value"),h.index("ID")
per=collections.defaultdict(dict); name={}
for r in rows[hi+1:]:
    if len(r)>iv: per[int(r[iid])][r[im]]=float(r[iv].replace(',','')); name[int(r[iid])]=r[ik].split('(')[0].replace('void ','').replace('<unnamed>::','')
for k in sorted(per):
    if name[k].startswith('k_t'):
        m=per[k]; print(k, name[k][:28], round(m.get('gpu__time_duration.sum',0)/1e3,1),'us', round((m.get('dram__bytes_read.sum',0)+m.get('dram__bytes_write.sum',0))/1e6,1),'MB', round(m.get('smsp__inst_executed.sum',0)/1e6,1),'Minst')
PY
