import sys; sys.path.insert(0, '.')
from paper_conf_cluster_ajipbf15_b200 import mcl
names = {0: "VIMNMX", 1: "VIMNMX3", 2: "IADD3", 3: "IMAD", 4: "VIMNMX3+IMAD", 5: "IMAD.HI", 6: "VIMNMX + FMA-pipe max"}
for op in range(7):
    r, c, m = mcl.mcl_probe_int_rate(0, op)
    print(f"op {op} {names[op]:24s} {r:.4e} lane-ops/s {c:6.2f} lane-ops/clk/SM  {m:.0f} MHz")
