#!/usr/bin/env python
"""Resolves preprocessor conditionals on fixed macro values (a minimal unifdef): A/B variant
switches that lost their measurement are folded to the winning value and their dead branches
removed.  Conditions naming any other macro are kept verbatim.

    python tools/unifdef.py FILE NAME=VALUE ...
"""
import re
import sys


def _eval(cond: str, vals: dict):
    names = set(re.findall(r"\b[A-Z_][A-Z0-9_]*\b", cond)) - {"defined"}
    if not names or not names <= set(vals):
        return None
    e = re.sub(r"defined\s*\(\s*(\w+)\s*\)", lambda m: "1", cond)
    for n in names:
        e = re.sub(rf"\b{n}\b", str(vals[n]), e)
    e = e.replace("&&", " and ").replace("||", " or ")
    e = re.sub(r"!(?!=)", " not ", e)
    return bool(eval(e))


def unifdef(lines, vals):
    out = []
    # stack entries: (mode, taken) -- mode "keep": emit the directives; "fold": resolved here
    stack = []
    emit = lambda: all(s[2] for s in stack)  # noqa: E731
    for ln in lines:
        s = ln.strip()
        m = re.match(r"#\s*(if|ifdef|ifndef|elif|else|endif)\b(.*)", s)
        if not m:
            if emit():
                out.append(ln)
            continue
        d, rest = m.group(1), m.group(2).strip()
        rest = re.sub(r"//.*$", "", rest).strip()
        if d in ("if", "ifdef", "ifndef"):
            if d == "ifdef":
                c = None if rest not in vals else True
            elif d == "ifndef":
                c = None if rest not in vals else False
            else:
                c = _eval(rest, vals)
            if c is None:
                stack.append(["keep", None, True])
                if emit():
                    out.append(ln)
            else:
                par = emit()
                stack.append(["fold", c, c])
                stack[-1][2] = c
                stack[-1].append(par)
        elif d == "elif":
            top = stack[-1]
            if top[0] == "keep":
                if emit():
                    out.append(ln)
            else:
                c = _eval(rest, vals)
                if c is None:
                    raise SystemExit(f"unresolvable #elif after a folded #if: {s}")
                top[2] = (not top[1]) and c
                top[1] = top[1] or c
        elif d == "else":
            top = stack[-1]
            if top[0] == "keep":
                if emit():
                    out.append(ln)
            else:
                top[2] = not top[1]
        else:  # endif
            top = stack.pop()
            if top[0] == "keep" and emit():
                out.append(ln)
    return out


def main():
    path, defs = sys.argv[1], sys.argv[2:]
    vals = {}
    for d in defs:
        k, v = d.split("=")
        vals[k] = int(v)
    lines = open(path).read().split("\n")
    res = unifdef(lines, vals)
    open(path, "w").write("\n".join(res))


if __name__ == "__main__":
    main()
