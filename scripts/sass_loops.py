"""List the loops (backward branches) of a kernel in a cuobjdump -sass dump with their size and
instruction mix:  python scripts/sass_loops.py dump.sass <function-substring> [min_size]"""
import collections, re, sys
txt = open(sys.argv[1]).read()
key = sys.argv[2]
mins = int(sys.argv[3]) if len(sys.argv) > 3 else 100
funcs = re.split(r"\n\s*Function : ", txt)
for f in funcs[1:]:
    name = f.split("\n", 1)[0]
    if key not in name:
        continue
    ins = []
    for line in f.split("\n"):
        m = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*?)\s*;", line)
        if m:
            ins.append((int(m.group(1), 16), m.group(2)))
    addr = {a: i for i, (a, _) in enumerate(ins)}
    print(name, len(ins), "instructions")
    for i, (a, s) in enumerate(ins):
        m = re.search(r"BRA (?:`\(\.L_x_\d+\) )?0x([0-9a-f]+)", s) or re.search(r"BRA\s+0x([0-9a-f]+)", s)
        if m:
            tgt = int(m.group(1), 16)
            if tgt < a and tgt in addr and i - addr[tgt] >= mins:
                body = [x for _, x in ins[addr[tgt]:i + 1]]
                ops = collections.Counter(re.sub(r"^@!?U?P\w+\s+", "", x).split()[0].split(".")[0] for x in body)
                print(f"  loop {tgt:#x}..{a:#x}: {len(body)} instr  " + " ".join(f"{k}:{v}" for k, v in ops.most_common(14)))
