"""Summarise `ptxas -v` output: one line per function (registers, stack,
spill bytes).  Usage: python tools/ptxas_summary.py build.log [filter]"""
import re
import sys

info, order, cur = {}, [], None
for line in open(sys.argv[1]):
    line = line.strip()
    m = re.search(r"(?:Compiling entry function|Function properties for) '?([^' ]+)'?", line)
    if m:
        cur = m.group(1)
        if cur not in info:
            info[cur] = {}
            order.append(cur)
        continue
    m = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads", line)
    if m and cur:
        info[cur].update(stack=int(m.group(1)), st=int(m.group(2)), ld=int(m.group(3)))
        continue
    m = re.search(r"Used (\d+) registers", line)
    if m and cur:
        info[cur]["regs"] = int(m.group(1))
flt = sys.argv[2] if len(sys.argv) > 2 else ""
for name in order:
    r = info[name]
    n = re.sub(r"__nv_static_\d+__\w+?_cu_\w+?_\d+__ZN\d+_GLOBAL__N__\w+?_cu_\w+?_\d+", "", name)
    if flt in n:
        print(f"{r.get('regs', 0):4d} regs {r.get('stack', 0):5d} stack "
              f"{r.get('st', 0):5d}/{r.get('ld', 0):5d} spill  {n[:100]}")
