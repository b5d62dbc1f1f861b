import csv, sys
for f in sys.argv[1:]:
    rows=[r for r in csv.reader(open(f)) if r and (r[0]=="ID" or r[0].isdigit())]
    h=rows[0]; ik=h.index("Kernel Name"); im=h.index("Metric Name"); iv=h.index("Metric Value"); ii=h.index("ID")
    agg={}
    for r in rows[1:]:
        agg.setdefault((r[ii],r[ik][:40]),{})[r[im]]=r[iv]
    print(f); tot=0
    for (i,k),m in list(agg.items())[-6:]:
        t=float(m['gpu__time_duration.sum'].replace(',',''))/1e3; tot+=t
        print(f"  {k:40s} {t:8.1f} us  rd {float(m['dram__bytes_read.sum'].replace(',',''))/1e9:6.2f} GB wr {float(m['dram__bytes_write.sum'].replace(',',''))/1e9:6.2f} GB")
    print("  total", round(tot,1))
