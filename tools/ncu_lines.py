"""Summarise an ncu report: headline metrics + hottest source lines.
usage: python tools/ncu_lines.py REPORT.ncu-rep [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
hdr = r[0]
want = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'lts__t_sector_hit_rate.pct', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'launch__registers_per_thread', 'lts__t_sectors.sum', 'smsp__inst_executed.sum',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'launch__grid_size']
for row in r[2:]:
    print(" | ".join(f"{w.split('.')[0]}={row[hdr.index(w)]}" for w in want if w in hdr))
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source=cuda,sass"],
                     capture_output=True, text=True).stdout
res = []; f = None; tot = 0; totw = 0
for x in csv.reader(io.StringIO(src)):
    if x and x[0] == 'File Path':
        f = x[1].split('/')[-1]; continue
    if len(x) < 9 or x[0] in ('Line No', ''):
        continue
    try:
        I = float(x[7]); W = float(x[4]); T = float(x[8])
    except ValueError:
        continue
    res.append((f, x[0], x[1][:90], I, W, T)); tot += I; totw += W
print('total warp inst %.3g, stall samples %d' % (tot, totw))
for x in sorted(res, key=lambda x: -x[4])[:top]:
    print('%-18s %4s inst %.3f stall %.3f thr/inst %4.1f  %s' % (x[0], x[1], x[3] / tot, x[4] / max(1, totw),
                                                             x[5] / max(1, x[3]), x[2]))
if len(sys.argv) > 3:
    # instruction share per line range "a-b,c-d" of the first file
    for rg in sys.argv[3].split(','):
        a, b = map(int, rg.split('-'))
        I = sum(x[3] for x in res if x[0] == 'gb_msbfs.cu' and a <= int(x[1]) <= b)
        W = sum(x[4] for x in res if x[0] == 'gb_msbfs.cu' and a <= int(x[1]) <= b)
        print(f"lines {a}-{b}: inst {I / tot:.3f} stall {W / max(1, totw):.3f}")
