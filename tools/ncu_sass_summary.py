import csv, subprocess, sys
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines())); h = r[0]; v = r[2]
want = ['gpu__time_duration.sum','dram__bytes_read.sum','dram__bytes_write.sum','sm__warps_active.avg.pct_of_peak_sustained_active','launch__registers_per_thread','launch__grid_size','launch__occupancy_limit_registers','smsp__inst_executed.sum','lts__t_sector_hit_rate.pct','lts__t_sectors.sum','smsp__thread_inst_executed_per_inst_executed.ratio']
print({w: v[h.index(w)] for w in want if w in h})
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(src.splitlines()))
hh = rows[1]; data = rows[2:]
iS = hh.index("Warp Stall Sampling (All Samples)"); iE = hh.index("Instructions Executed"); iSrc = hh.index("Source"); iA = hh.index("Address")
tot = sum(float(x[iS] or 0) for x in data); te = sum(float(x[iE] or 0) for x in data)
print("total samples", tot, "inst", te)
for x in sorted(data, key=lambda x: -float(x[iS] or 0))[:int(sys.argv[2]) if len(sys.argv) > 2 else 14]:
    print(x[iA][-5:], x[iSrc][:70].ljust(70), x[iS], x[iE])
