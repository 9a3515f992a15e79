"""Decode the scheduling control bits (stall, yield, write/read scoreboard, wait mask) of
the SASS of one kernel (Volta+ encoding: bits 41..61 of the high 64-bit word).
Usage: sass_ctrl.py lib.so mangled_kernel_name [start_hex end_hex]"""
import re, subprocess, sys
so, fn = sys.argv[1], sys.argv[2]
lo = int(sys.argv[3], 16) if len(sys.argv) > 3 else 0
hi = int(sys.argv[4], 16) if len(sys.argv) > 4 else 1 << 40
out = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True).stdout
funcs = re.split(r"\n\s+Function : ", out)
body = [f for f in funcs if f.startswith(fn)][0].split("\n")
i = 0
while i < len(body):
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?);\s*/\* (0x[0-9a-f]+) \*/", body[i])
    if m and i + 1 < len(body):
        m2 = re.search(r"/\* (0x[0-9a-f]+) \*/", body[i + 1])
        addr, txt = int(m.group(1), 16), m.group(2).strip()
        h = int(m2.group(1), 16)
        stall = (h >> 41) & 0xF
        yld = (h >> 45) & 1
        wb = (h >> 46) & 7
        rb = (h >> 49) & 7
        wm = (h >> 52) & 0x3F
        if lo <= addr <= hi:
            w = "".join(str(k) for k in range(6) if wm >> k & 1)
            print(f"{addr:#06x} S{stall:02d} {'Y' if yld else ' '} W{wb if wb != 7 else '-'} R{rb if rb != 7 else '-'} wait[{w:6s}] {txt}")
        i += 2
    else:
        i += 1
