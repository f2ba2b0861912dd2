"""Key metrics, warp-state samples and per-cell instruction mix of two ncu --set full
captures (developer tool): python tools/ncu_final_summary.py <headline.ncu-rep> <rows_blocks.ncu-rep>"""
import csv, subprocess, sys, collections
def raw(rep):
    out = subprocess.run(["ncu","-i",rep,"--page","raw","--csv"],capture_output=True,text=True).stdout
    r = list(csv.reader(out.splitlines())); return {k: (v + " " + u).strip() for k, u, v in zip(r[0], r[1], r[2])}
def mix(rep, cells):
    out = subprocess.run(["ncu","-i",rep,"--page","source","--csv","--print-source","sass"],capture_output=True,text=True).stdout
    rows = list(csv.reader(out.splitlines())); h=rows[1]; data=rows[2:]
    iS=h.index('Source'); iE=h.index('Instructions Executed')
    c=collections.Counter(); tot=0
    for r in data:
        op=r[iS].strip().split()
        if not op: continue
        o=op[1] if op[0].startswith('@') else op[0]; o=o.split('.')[0]
        n=int(r[iE] or 0); c[o]+=n; tot+=n
    return tot*32/cells, c
for name, rep, cells in [("dfg_fused_tma, fused Q 1024^3 fp32 (bench headline)", sys.argv[1], 1024**3),
                         ("dfg_fused_rows_multi, 12 packed VisIt blocks 192x192x256 (bench visit_blocks)", sys.argv[2], 12*192*192*256)]:
    d = raw(rep)
    g = lambda k: d.get(k, "")
    print(f"### {name}\n")
    print("| metric | value |\n|---|---|")
    for k, lab in [("gpu__time_duration.sum","duration (ncu clocks)"),("sm__cycles_elapsed.avg.per_second","SM clock"),
                   ("dram__bytes_read.sum","DRAM read"),("dram__bytes_write.sum","DRAM write"),
                   ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed","DRAM throughput (of ncu peak)"),
                   ("sm__inst_issued.avg.pct_of_peak_sustained_active","issue slots busy"),
                   ("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed","L1 data pipe (elapsed)"),
                   ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum","shared bank conflicts"),
                   ("launch__registers_per_thread","registers"),("launch__block_size","threads per CTA"),("launch__grid_size","CTAs")]:
        print(f"| {lab} | {g(k)} |")
    ipc, c = mix(rep, cells)
    print(f"| thread instructions per cell | {ipc:.1f} |")
    st = {k.replace('smsp__pcsamp_warps_issue_stalled_',''): int(float(d[k].split()[0])) for k in d if k.startswith('smsp__pcsamp_warps_issue_stalled') and not k.endswith('not_issued')}
    tot = sum(st.values()) or 1
    print("\nwarp-state samples: " + ", ".join(f"{k} {100*v/tot:.0f} %" for k,v in sorted(st.items(), key=lambda x:-x[1])[:7]))
    print("\ninstructions per cell: " + ", ".join(f"{o} {n*32/cells:.2f}" for o,n in c.most_common(14)) + "\n")
