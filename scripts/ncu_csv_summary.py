"""Per-launch summary of an `ncu --metrics ... --csv` log (gpu time, L1 global-load sectors, DRAM
bytes per requested sector, L2 sectors per L1 sector, L2 hit rate).
usage: python scripts/ncu_csv_summary.py launches.csv"""
import sys,csv,collections
rows=[r for r in csv.reader(l for l in open(sys.argv[1]) if l.startswith('"'))]
h=rows[0]; k=collections.OrderedDict()
for r in rows[1:]:
    d=dict(zip(h,r))
    if d['Metric Value']=='n/a': continue
    k.setdefault((d['ID'],d['Kernel Name'][:30]),{})[d['Metric Name']]=float(d['Metric Value'].replace(',',''))
for (i,n),m in k.items():
    t=m['gpu__time_duration.sum']*1e-9
    sec=m['l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum']; req=m['l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum']
    dram=m['dram__bytes_read.sum']+m['dram__bytes_write.sum']
    lts=m['lts__t_sectors_srcunit_tex_op_read.sum']
    print(f"{i:>3} {n:30s} t={t*1e3:8.3f}ms L1sec={sec:.3e} ({sec/t:.2e}/s) dram={dram/t/1e12:.2f}TB/s dramB/L1sec={dram/sec:.1f} lts/L1sec={lts/sec:.2f} hit={m['lts__t_sector_op_read_hit_rate.pct']:.1f}%")
