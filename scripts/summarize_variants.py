"""profiles/ncu_variants_r1.txt from gpurun_out/variants.csv + variants.log (scripts/prof_variants.py)."""
import csv, sys
rows = list(csv.reader(open('gpurun_out/variants.csv')))
hi = [i for i, r in enumerate(rows) if r and r[0] == 'ID'][0]
hdr, data = rows[hi], rows[hi + 1:]
I = {h: i for i, h in enumerate(hdr)}
labels = [l.split()[1:] for l in open('gpurun_out/variants.log') if l.startswith('launch ')]
per, order = {}, []
for r in data:
    k = r[I['ID']]
    if k not in per:
        per[k] = {}
        order.append(k)
    per[k][r[I['Metric Name']]] = (r[I['Metric Value']], r[I['Metric Unit']])
SC = {'byte': 1e-6, 'Kbyte': 1e-3, 'Mbyte': 1.0, 'Gbyte': 1e3, 'ns': 1e-3, 'us': 1.0, 'usecond': 1.0, 'ms': 1e3,
      'msecond': 1e3, 'nsecond': 1e-3}
def g(d, m):
    if m not in d:
        return float('nan')
    v, u = d[m]
    try:
        v = float(v.replace(',', ''))
    except ValueError:
        return float('nan')
    return v * SC.get(u, 1.0)
out = ["per-variant ncu (ncu --metrics $(cat scripts/prof_variants_metrics.txt) --clock-control none -k regex:'spmv_claim_kernel|sgemm_'; "
       "scripts/prof_variants.py: each pool variant's pure full-grid kernel once; cold caches, serialised replays)",
       "FMA% / TC% = sm__pipe_fma_cycles_active / sm__pipe_tensor_cycles_active .avg.pct_of_peak_sustained_active",
       f"{'config':16s} {'variant':18s} {'us':>9s} {'DRAM rd MB':>10s} {'wr MB':>7s} {'DRAM%':>6s} {'L2hit%':>6s} "
       f"{'L1TEX%':>6s} {'FMA%':>6s} {'TC%':>6s} {'grid':>6s} {'regs':>4s}"]
for k, lab in zip(order, labels):
    d = per[k]
    out.append(f"{lab[0]:16s} {lab[1]:18s} {g(d,'gpu__time_duration.sum'):9.1f} {g(d,'dram__bytes_read.sum'):10.1f} "
               f"{g(d,'dram__bytes_write.sum'):7.1f} {g(d,'dram__throughput.avg.pct_of_peak_sustained_elapsed'):6.1f} "
               f"{g(d,'lts__t_sector_hit_rate.pct'):6.1f} {g(d,'l1tex__throughput.avg.pct_of_peak_sustained_active'):6.1f} "
               f"{g(d,'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active'):6.1f} "
               f"{g(d,'sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active'):6.1f} "
               f"{g(d,'launch__grid_size'):6.0f} {g(d,'launch__registers_per_thread'):4.0f}")
open('profiles/ncu_variants_r1.txt', 'w').write("\n".join(out) + "\n")
print("\n".join(out))
