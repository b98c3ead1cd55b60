"""CPU oracle for the profile CSV ingest (NEXT-4) -- TEST INFRASTRUCTURE ONLY.

PAPER.md P:59 / P:65: the profiler records, per kernel invocation, the kernel name, the dynamic
instruction count and the CTA count (Sieve's inputs); "the output of which is converted
into a readable CSV file which serves as input to the Sieve sampling methodology".  The paper
does not fix the CSV dialect; reading A27 does:
  * one row per invocation in launch order; `header_lines` leading lines are skipped;
  * fields separated by `delimiter`; double quotes toggle quoting (a quoted field may hold the
    delimiter); the quote characters themselves are not part of the value;
  * numeric fields may carry thousands separators (',', '_') and padding (' ', '\\t');
  * a line ending in '\\r\\n' loses the '\\r'; the last line may lack its '\\n';
  * kernel names are interned into dense ids in order of first appearance.
This is the plain definition, written with Python's str operations, row by row.
"""


def _fields(line, delim):
    out, cur, inq = [], [], False
    for ch in line:
        if ch == '"':
            inq = not inq
        elif ch == delim and not inq:
            out.append("".join(cur))
            cur = []
        else:
            cur.append(ch)
    out.append("".join(cur))
    return out


def _number(field):
    digits = [c for c in field if c not in ',"_ \r\t']
    if not digits or any(not ("0" <= c <= "9") for c in digits):
        raise ValueError(f"not a non-negative integer: {field!r}")
    v = int("".join(digits))
    if v >= 1 << 64:
        raise ValueError("value does not fit 64 bits")
    return v


def parse(text, col_kernel, col_instr, col_cta=-1, col_cycles=-1, header_lines=1, delimiter=","):
    """-> (kernel_id, instr, cta | None, cycles | None, names) as Python lists."""
    lines = text.split("\n") if text else []
    if text.endswith("\n"):
        lines = lines[:-1]
    rows = lines[header_lines:]
    ids, names = {}, []
    kid, x, cta, y = [], [], [], []
    for line in rows:
        if line.endswith("\r"):
            line = line[:-1]
        f = _fields(line, delimiter)
        need = max(col_kernel, col_instr, col_cta, col_cycles)
        if len(f) <= need:
            raise ValueError(f"row has {len(f)} fields, needs {need + 1}")
        name = f[col_kernel]
        if name not in ids:
            ids[name] = len(names)
            names.append(name)
        kid.append(ids[name])
        x.append(_number(f[col_instr]))
        if col_cta >= 0:
            c = _number(f[col_cta])
            if c >= 1 << 32:
                raise ValueError("CTA count does not fit 32 bits")
            cta.append(c)
        if col_cycles >= 0:
            y.append(_number(f[col_cycles]))
    return kid, x, (cta if col_cta >= 0 else None), (y if col_cycles >= 0 else None), names


def write(kid, x, cta, cycles, names, delimiter=",", thousands=False, crlf=False, trailing=True,
          header="ID,Kernel Name,Instructions,CTAs,Cycles"):
    """Render a trace as profiler-style CSV text (test input builder; no method arithmetic)."""
    nl = "\r\n" if crlf else "\n"
    fmt = (lambda v: f'"{v:,}"') if thousands else (lambda v: str(v))
    out = [header]
    for i in range(len(kid)):
        row = [str(i), '"' + names[kid[i]] + '"', fmt(int(x[i]))]
        row.append(fmt(int(cta[i])) if cta is not None else "0")
        row.append(fmt(int(cycles[i])) if cycles is not None else "0")
        out.append(delimiter.join(row))
    return nl.join(out) + (nl if trailing else "")
