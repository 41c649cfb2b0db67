import re, sys
txt = open(sys.argv[1]).read()
txt = txt.split("=== FWD ===")[-1].split("=== END ===")[0]
rt = re.findall(r"RTTRACE start (\d+)", txt)
rte = re.findall(r"RTTRACE tail_start (\d+) end (\d+)", txt)
units = [dict(zip(["cta","sm","grp","exp","chunk","n","in","unit","a","b"], map(int, m))) for m in
         re.findall(r"FDTRACE cta (\d+) sm (\d+) grp (\d+) exp (-?\d+) chunk (\d+) n (\d+) in (\d+) unit (\d+) a_done (\d+) b_done (\d+)", txt)]
t0 = int(rt[0]) if rt else min(u["in"] for u in units)
print("route start 0, tail start %.1f us, route end %.1f us" % ((int(rte[0][0]) - t0) / 1e3, (int(rte[0][1]) - t0) / 1e3) if rte else "no route trace")
print("units", len(units))
for key in ["in", "unit", "a", "b"]:
    v = sorted((u[key] - t0) / 1e3 for u in units)
    print(f"{key:5s} min {v[0]:7.1f} p10 {v[len(v)//10]:7.1f} med {v[len(v)//2]:7.1f} p90 {v[9*len(v)//10]:7.1f} max {v[-1]:7.1f}")
pa = sorted((u["a"] - u["unit"]) / 1e3 for u in units); pb = sorted((u["b"] - u["a"]) / 1e3 for u in units)
print("phaseA dur med %.1f max %.1f | phaseB dur med %.1f max %.1f" % (pa[len(pa)//2], pa[-1], pb[len(pb)//2], pb[-1]))
sh = [u for u in units if u["grp"] == 1]
if sh:
    print("shared units: A done med %.1f, B done max %.1f" % (sorted((u["a"]-t0)/1e3 for u in sh)[len(sh)//2], max((u["b"]-t0)/1e3 for u in sh)))
