"""Summarise build/ptxas.log: registers / spills per kernel (dev helper)."""
import re
import sys

log = open(sys.argv[1] if len(sys.argv) > 1 else "paper_conf_sc_zhengspl25_b200/build/ptxas.log").read()
for blk in log.split("Compiling entry function")[1:]:
    name = re.search(r"'(\S+)'", blk).group(1)
    m = re.search(r"(\w+kernel)\w*?(I[^E]*E)?", name)
    short = name[name.find("kernel") - 10:][:60] if "kernel" in name else name[:60]
    regs = re.search(r"Used (\d+) registers", blk)
    sp = re.search(r"(\d+) bytes spill stores, (\d+) bytes spill loads", blk)
    print(f"{short:62s} regs={regs.group(1) if regs else '?':>4} spill_st={sp.group(1) if sp else '?'} spill_ld={sp.group(2) if sp else '?'}")
