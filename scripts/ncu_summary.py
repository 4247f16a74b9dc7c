"""Condense an ncu --set full report into profiles/<name>_ncu_details.json and write
profiles/traffic_latest.json (DRAM bytes per sample of each sampling kernel).
usage: python scripts/ncu_summary.py report.ncu-rep out.json samples_per_launch"""
import csv
import io
import json
import subprocess
import sys

rep, out_path, samples = sys.argv[1], sys.argv[2], float(sys.argv[3])
WORKLOAD = ("C1: eu2005-shaped Chung-Lu power-law graph, |V|=862664, |E|=16138468, unlabelled; "
            "dense 8-vertex random-walk query (seed 21); WanderJoin + Alley, 1e8 samples each per step")


def page(p):
    txt = subprocess.run(["ncu", "-i", rep, "--page", p, "--csv"], capture_output=True, text=True).stdout
    return list(csv.reader(io.StringIO(txt)))


def kname(s):
    s = s.split("(")[0]
    return "wj" if "sample_kernel<0" in s else "alley" if "sample_kernel<1" in s else s


keep = ['Duration', 'Elapsed Cycles', 'SM Frequency', 'DRAM Throughput', 'Memory Throughput', 'L1/TEX Hit Rate',
        'L2 Hit Rate', 'Compute (SM) Throughput', 'Issue Slots Busy', 'Executed Ipc Active',
        'Avg. Active Threads Per Warp', 'Achieved Occupancy', 'Theoretical Occupancy', 'Registers Per Thread',
        'Grid Size', 'Block Size', 'Warp Cycles Per Issued Instruction', 'Eligible Warps Per Scheduler',
        'No Eligible', 'Branch Efficiency']
rows = page("details")
hdr = rows[0]
out = {}
for r in rows[1:]:
    n = r[hdr.index('Metric Name')]
    if n in keep:
        out.setdefault(kname(r[4]), {})[n] = r[hdr.index('Metric Value')] + ' ' + r[hdr.index('Metric Unit')]
raw = page("raw")
h, units = raw[0], raw[1]
want = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum', 'lts__t_sectors.sum',
        'lts__t_sector_hit_rate.pct', 'smsp__thread_inst_executed_per_inst_executed.ratio',
        'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum', 'l1tex__throughput.avg.pct_of_peak_sustained_active',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed']
scale = {'Gbyte': 1e9, 'Mbyte': 1e6, 'Kbyte': 1e3, 'byte': 1.0, 'Tbyte': 1e12}
traffic = {}
for r in raw[2:]:
    k = kname(r[h.index('Kernel Name')])
    for w in want:
        if w in h:
            out.setdefault(k, {})[w] = r[h.index(w)] + ' ' + units[h.index(w)]
    tb = sum(float(r[h.index(w)].replace(',', '')) * scale[units[h.index(w)]]
             for w in ('dram__bytes_read.sum', 'dram__bytes_write.sum'))
    traffic[k] = tb / samples
out['_capture'] = {'report': rep, 'samples_per_launch': samples, 'workload': WORKLOAD}
json.dump(out, open(out_path, 'w'), indent=1)


def num(k, key):
    v = out.get(k, {}).get(key)
    return float(v.split()[0].replace(',', '')) if v else None


# the counters the north star asks the design to be backed by, per sampling kernel
counters = {}
for k in ('wj', 'alley'):
    if k not in out:
        continue
    counters[k] = {
        "achieved_occupancy_pct": num(k, 'Achieved Occupancy'),
        "active_threads_per_warp_instruction": num(k, 'smsp__thread_inst_executed_per_inst_executed.ratio'),
        "warp_execution_efficiency": (num(k, 'smsp__thread_inst_executed_per_inst_executed.ratio') or 0) / 32.0,
        "issue_slots_busy_pct": num(k, 'Issue Slots Busy'),
        "eligible_warps_per_scheduler": num(k, 'Eligible Warps Per Scheduler'),
        "l2_hit_rate_pct": num(k, 'lts__t_sector_hit_rate.pct'),
        "l1_global_load_sectors_per_sample": (num(k, 'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum') or 0) / samples,
        "l2_sectors_per_sample": (num(k, 'lts__t_sectors.sum') or 0) / samples,
        "dram_sectors_per_sample": traffic.get(k, 0.0) / 32.0,
        # no unit saturated: L1TEX and L2 throughput against their peaks
        "l1tex_throughput_pct": num(k, 'l1tex__throughput.avg.pct_of_peak_sustained_active'),
        "lts_throughput_pct": num(k, 'lts__throughput.avg.pct_of_peak_sustained_elapsed'),
        "shared_wavefronts_pct": num(k, 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed'),
    }
json.dump({"workload": WORKLOAD, "captured_samples_per_launch": samples, "dram_bytes_per_sample": traffic,
           "counters": counters,
           "source": out_path + " (ncu --set full; dram__bytes_read.sum + dram__bytes_write.sum)"},
          open("profiles/traffic_latest.json", "w"), indent=1)
print(json.dumps(out, indent=1))
