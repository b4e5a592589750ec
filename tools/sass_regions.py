"""Static per-region SASS instruction counts of the built kernels (no GPU).

The warp simulator (oracle/warpsim.c) counts, per source region of the hot
path, warp executions and active lanes.  SIMT efficiency needs the
cost of each region in SASS instructions; this tool reads it off the cubin in
libsr.so:

  * regions are delimited in the CUDA source by `// @sr-region NAME[:full]`
    comments (a marker applies from its line to the next marker);
  * every SASS instruction is attributed to the innermost frame of its inline
    chain (nvdisasm -gi) that lies in a marked region (so a marked device
    function such as the MC step splits into its own regions, while unmarked
    helpers such as Philox count toward their call site);
  * cold code is excluded: the slow path of BRA.DIV (WARPSYNC.COLLECTIVE
    sequences), the trailing self-branch/NOP padding, and subroutines reached
    by CALL.REL (IEEE div/sqrt slow paths);
  * a CALL.ABS to a non-inlined device function (foo of config 2) adds the
    callee's instruction count to the calling region.

`:full` marks code executed by every valid lane of the warp whenever the
region's scheduler step runs (round bookkeeping, branch headers), as opposed
to the lanes the simulator puts in that region's mask.

usage: python tools/sass_regions.py [kernel-regex]   -> JSON on stdout
"""
from __future__ import annotations

import json
import os
import re
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_cgo_damanijskymg20_b200", "libsr.so")
CSRC = os.path.join(ROOT, "paper_conf_cgo_damanijskymg20_b200", "csrc")

LINE_RE = re.compile(r'//## File "([^"]+)", line (\d+)(.*)')
INL_RE = re.compile(r'inlined at "([^"]+)", line (\d+)')
INS_RE = re.compile(r"/\*([0-9a-f]{4,})\*/\s+(.*?)\s*;")
MARK_RE = re.compile(r"//\s*@sr-region\s+([A-Z_0-9]+)(:full)?")


def region_map(path):
    """line -> (region, full) from the @sr-region markers of one source file."""
    out, cur = {}, None
    for i, line in enumerate(open(path), 1):
        m = MARK_RE.search(line)
        if m:
            cur = None if m.group(1) == "END" else (m.group(1), bool(m.group(2)))
        if cur is not None:
            out[i] = cur
    return out


def marked_call_lines(path):
    """Lines that call a __device__ function whose own body carries markers
    (e.g. the MC step): an instruction resolved only to such a line lost its
    intermediate inline frames."""
    src = open(path).read().splitlines()
    fn, marked, body = None, set(), {}
    for line in src:
        m = re.search(r"__device__[^(;]*?\b(\w+)\s*\(", line)
        if m and "__global__" not in line:
            fn = m.group(1)
        elif "__global__" in line:
            fn = None
        if fn:
            body.setdefault(fn, []).append(line.split("//")[0])
            if MARK_RE.search(line):
                marked.add(fn)
    # transitively: a function calling a marked function (MC step -> step_a/b)
    changed = True
    while changed:
        changed = False
        for f, lines in body.items():
            if f not in marked and any(re.search(r"\b%s\s*(?:<[^<>()]*>)?\s*\(" % g, c)
                                       for g in marked for c in lines[1:]):
                marked.add(f)
                changed = True
    out = set()
    for i, line in enumerate(src, 1):
        code = line.split("//")[0]
        if any(re.search(r"\b%s\s*(?:<[^<>()]*>)?\s*\(" % f, code) for f in marked) and \
                "__device__" not in code:
            out.add(i)
    return out


def extract_cubins(tmp):
    subprocess.run(["cuobjdump", "-xelf", "all", LIB], cwd=tmp, capture_output=True)
    return [os.path.join(tmp, f) for f in os.listdir(tmp) if f.endswith(".cubin")]


def _parse(txt):
    funcs, cur, loc, labels = {}, None, (None, None, []), []
    for raw in txt.splitlines():
        m = re.match(r"\s*\.text\.(\S+):", raw)
        if m:
            cur = m.group(1)
            funcs[cur] = []
            continue
        if cur is None:
            continue
        m = LINE_RE.search(raw)
        if m:
            f, ln, rest = m.group(1), int(m.group(2)), m.group(3)
            loc = (f, ln, [(f, ln)] + [(a, int(b)) for a, b in INL_RE.findall(rest)])
            continue
        m = re.match(r"^(\.L_x_\d+|\$\S+):$", raw.strip())
        if m:
            labels.append(m.group(1))
            continue
        m = INS_RE.search(raw)
        if m:
            funcs[cur].append(dict(addr=int(m.group(1), 16), text=m.group(2), file=loc[0],
                                   line=loc[1], frames=loc[2], labels=labels))
            labels = []
    return funcs


def parse_functions(cubin):
    """{function: [dict(addr, text, chain, labels)]}.  nvdisasm -g gives the
    innermost source line of every instruction; -gi adds one 'inlined at'
    frame (and for deeper inlining reports an outer call site instead), so the
    chain is the -g frame followed by the -gi frames."""
    g = _parse(subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True,
                              text=True).stdout)
    gi = _parse(subprocess.run(["nvdisasm", "-gi", "-c", cubin], capture_output=True,
                               text=True).stdout)
    out = {}
    for name, ins in g.items():
        other = gi.get(name, [])
        for k, x in enumerate(ins):
            chain = list(x["frames"][:1])
            if k < len(other) and other[k]["addr"] == x["addr"]:
                chain += [fr for fr in other[k]["frames"] if fr not in chain]
            x["chain"] = chain
        out[name] = ins
    return out


def basic_blocks(ins):
    """[start, end) index ranges: a block starts at a label or after a branch."""
    bbs, start = [], 0
    for i, x in enumerate(ins):
        if i > start and x["labels"]:
            bbs.append((start, i))
            start = i
        if re.match(r"(@!?U?P\w+\s+)?(BRA|EXIT|RET)\b", x["text"]):
            bbs.append((start, i + 1))
            start = i + 1
    if start < len(ins):
        bbs.append((start, len(ins)))
    return bbs


def cold_set(ins):
    """Indices of instructions on cold paths."""
    label_at = {}
    for i, x in enumerate(ins):
        for lb in x["labels"]:
            label_at[lb] = i
    cold = set()
    # 1. BRA.DIV slow paths and CALL.REL subroutines: from the target label up
    #    to (and including) the block's terminating branch back / RET
    starts = []
    for x in ins:
        m = re.search(r"BRA\.DIV\s+\S+,\s*`\((\.L_x_\d+)\)", x["text"])
        if m:
            starts.append(m.group(1))
    for lb in starts:
        i = label_at.get(lb)
        while i is not None and i < len(ins):
            cold.add(i)
            t = ins[i]["text"]
            if re.match(r"(@\S+\s+)?(RET|BRA)\b", t) and not t.startswith("@"):
                break
            i += 1
    # 2. the argument/result moves around a call of a cold subroutine (the IEEE
    #    div/sqrt slow paths): the whole basic block holding the CALL is cold
    for a, b in basic_blocks(ins):
        if any(re.search(r"CALL\.\w+(?:\.NOINC)?\s+`\(\$__internal", ins[i]["text"])
               for i in range(a, b)):
            cold.update(range(a, b))
    # 3. trailing trap loop / padding
    for i, x in enumerate(ins):
        m = re.search(r"BRA\s+`\((\.L_x_\d+)\)", x["text"])
        if m and label_at.get(m.group(1)) == i:
            cold.update(range(i, len(ins)))
            break
    return cold


def loop_intervals(ins):
    """[start, end] index ranges of loops (a branch back to an earlier label)."""
    label_at = {}
    for i, x in enumerate(ins):
        for lb in x["labels"]:
            label_at[lb] = i
    out = []
    for i, x in enumerate(ins):
        m = re.search(r"\bBRA\b.*`\((\.L_x_\d+)\)", x["text"])
        if m and "BRA.DIV" not in x["text"]:
            j = label_at.get(m.group(1))
            if j is not None and j < i:
                out.append((j, i))
    return out


def kernel_hashes(kernel_regex=".*"):
    """{kernel: sha256 of its SASS instruction text} -- identifies the exact
    code a stored ncu measurement belongs to."""
    import hashlib
    with tempfile.TemporaryDirectory() as tmp:
        out = {}
        for c in extract_cubins(tmp):
            txt = subprocess.run(["cuobjdump", "-sass", c], capture_output=True, text=True).stdout
            cur, buf = None, []
            for line in txt.splitlines() + ["Function : <end>"]:
                m = re.search(r"Function : (\S+)", line)
                if m:
                    if cur and re.search(kernel_regex, cur):
                        out[cur] = hashlib.sha256("\n".join(buf).encode()).hexdigest()[:16]
                    cur, buf = m.group(1), []
                else:
                    mm = re.search(r"/\*[0-9a-f]{4,}\*/\s+(.*?);", line)
                    if mm:
                        buf.append(mm.group(1).strip())
        return out


def kernel_costs(kernel_regex=".*"):
    maps, weak_lines = {}, set()
    for f in os.listdir(CSRC):
        if f.endswith(".cu"):
            path = os.path.join(CSRC, f)
            maps[path] = region_map(path)
            weak_lines |= {(path, ln) for ln in marked_call_lines(path)}
    with tempfile.TemporaryDirectory() as tmp:
        funcs = {}
        for c in extract_cubins(tmp):
            funcs.update(parse_functions(c))
    out = {}
    for name, ins in funcs.items():
        if not re.search(kernel_regex, name) or "foo" in name:
            continue
        # split the section: kernel body, then subroutines ($kernel$callee labels)
        subs, body_end = {}, len(ins)
        cur = None
        for i, x in enumerate(ins):
            for lb in x["labels"]:
                if lb.startswith("$"):
                    cur = lb
                    body_end = min(body_end, i)
                    subs[cur] = []
            if cur is not None:
                subs[cur].append(x)
        body = ins[:body_end]
        sub_size = {}
        for lb, si in subs.items():
            hot = "__internal" not in lb   # IEEE div/sqrt slow paths are cold
            sub_size[lb] = len(si) if hot else 0
        cold = cold_set(body)
        loops = [(a, b) for a, b in loop_intervals(body) if a not in cold and b not in cold]
        # region of each instruction: "strong" when resolved by its own line or
        # a reported call site; "weak" when only resolved by a line that calls
        # a marked device function (the intermediate call line was lost).
        # Weak instructions take the majority strong region of their basic
        # block (inlined helper code shares the block of its call site).
        strong, weak = [None] * len(body), [None] * len(body)
        for i, x in enumerate(body):
            ch = x["chain"]
            for j, (f, ln) in enumerate(ch):
                r = maps.get(f, {}).get(ln)
                if r is not None:
                    if j > 0 and (f, ln) in weak_lines:
                        weak[i] = r
                    else:
                        strong[i] = r
                    break
        bbs, start = [], 0
        for i, x in enumerate(body):
            if i > start and x["labels"]:
                bbs.append((start, i))
                start = i
            if re.match(r"(@!?U?P\w+\s+)?(BRA|EXIT|RET)\b", x["text"]) and \
                    not x["text"].startswith("BRA.DIV"):
                bbs.append((start, i + 1))
                start = i + 1
        if start < len(body):
            bbs.append((start, len(body)))
        nested = {i for a, b in loops for i in range(a, b + 1)
                  if any(a2 < a and b <= b2 or a2 <= a and b < b2 for a2, b2 in loops)}
        final, prev = [None] * len(body), None
        for a_, b_ in bbs:
            # predicated instructions are if-converted branch bodies: they say
            # which branch they came from, not which lanes run the block, so
            # only unpredicated instructions vote (unless there are none)
            votes, pvotes = {}, {}
            for i in range(a_, b_):
                # an entry-line special-register read or constant load inside a
                # nested loop is a rematerialisation (threadIdx, blockDim reloaded
                # where it is used, e.g. the path tracer's stack address in its
                # node-release loop): it says nothing about which region the block is in
                if strong[i] is not None and strong[i][0] == "ENTRY" and \
                        re.match(r"(S2R|S2UR|CS2R|LDC|LDCU|ULDC)\b", body[i]["text"]) and \
                        i in nested:
                    continue
                if strong[i] is not None and i not in cold:
                    d = pvotes if body[i]["text"].startswith("@") else votes
                    d[strong[i]] = d.get(strong[i], 0) + 1
            votes = votes or pvotes
            bb_reg = max(votes, key=votes.get) if votes else None
            for i in range(a_, b_):
                # every instruction of a basic block issues with the block's
                # mask (if-converted code and predicated-off lanes included), so
                # the block's majority region decides the lanes of all of them
                final[i] = bb_reg or strong[i] or prev or weak[i]
            if bb_reg is not None:
                prev = bb_reg
        # reconvergence points: the code at a BSSY's target label (and the BSYNC
        # that waits there) runs with the mask the warp had at the BSSY -- the
        # tail of an if/else that the compiler merged into the code after it
        # carries the line of one arm, but it issues for every lane that
        # entered the if, so it takes the region of the BSSY instruction
        label_blk = {}
        for k, (a_, b_) in enumerate(bbs):
            for lb in body[a_]["labels"]:
                label_blk[lb] = k
        # (in address order: a BSSY inside a block that was itself re-assigned
        # by an earlier reconvergence point reads its corrected region)
        blk_start = {a_: b_ for a_, b_ in bbs}
        open_bssy, pending = {}, {}
        for i, x in enumerate(body):
            if i in blk_start and i in pending:
                for j in range(i, blk_start[i]):
                    if not re.match(r"(?:@\S+\s+)?BSYNC", body[j]["text"]):
                        final[j] = pending[i]
            if i in cold:
                continue
            m = re.match(r"(?:@\S+\s+)?BSSY(?:\.\w+)?\s+(B\d+),\s*`\((\.L_x_\d+)\)", x["text"])
            if m and final[i] is not None:
                open_bssy[m.group(1)] = final[i]
                k = label_blk.get(m.group(2))
                if k is not None and bbs[k][0] > i:
                    pending[bbs[k][0]] = final[i]
                continue
            m = re.match(r"(?:@\S+\s+)?BSYNC(?:\.\w+)?\s+(B\d+)", x["text"])
            if m and m.group(1) in open_bssy:
                final[i] = open_bssy[m.group(1)]
        # loop nesting: a region whose code sits mostly in an inner loop (the merged
        # loop's partial unroll, the run-ahead loop, PDOM's inner do-while) may have
        # instructions the compiler hoisted into the enclosing loop; those run once
        # per entry of the inner loop -- per release / advance round / launch -- with
        # that step's lanes, so they are costed to the entering region
        regions_here = {f[0] for f in final if f is not None}
        # (the path tracer's PDOM traversal loop is entered once per bounce: BOUNCE)
        # (the path tracer's split merge: its node releases, NREL -- a simulator count)
        enter = {"STEP": ("BOUNCE" if "BOUNCE" in regions_here else
                          "RELEASE" if "RELEASE" in regions_here else
                          "NREL" if "REL" in regions_here else "LAUNCH"),
                 "PROLOG": "ADVANCE"}
        for rname, ename in enter.items():
            # (ADVANCE has no code of its own when the SCHED counters are compiled
            # out; the simulator still counts its rounds)
            if ename not in regions_here and ename not in ("LAUNCH", "ADVANCE", "NREL"):
                continue
            idx = [i for i in range(len(body)) if final[i] is not None and final[i][0] == rname
                   and i not in cold]
            if not idx:
                continue
            inner = [(a_, b_) for a_, b_ in loops
                     if sum(a_ <= i <= b_ for i in idx) * 2 > len(idx)]
            if ename == "NREL":
                # the split merge's node-release loop is the innermost loop holding most of
                # the NODE visits; the release's STEP code (loop entry / exit) lies outside it
                nidx = [i for i in range(len(body)) if final[i] is not None and
                        final[i][0] == "NODE" and i not in cold]
                inner = [(a_, b_) for a_, b_ in loops
                         if sum(a_ <= i <= b_ for i in nidx) * 2 > len(nidx)]
            if ename == "BOUNCE":
                # the path tracer's PDOM traversal loop (and the split merge's node-release
                # loop): its vote / latch are a few of the region's instructions, the loop's
                # entry and exit code the rest -- the innermost loop holding any of them is
                # the traversal loop
                inner = [(a_, b_) for a_, b_ in loops if any(a_ <= i <= b_ for i in idx)]
            if not inner:
                continue
            a_in, b_in = min(inner, key=lambda ab: ab[1] - ab[0])
            if not any(a_ < a_in and b_in < b_ for a_, b_ in loops):
                continue   # not nested: nothing can be hoisted out of it
            for i in idx:
                if not (a_in <= i <= b_in) and any(a_ <= i <= b_ for a_, b_ in loops):
                    final[i] = (ename, False)
        reg = {}
        unmapped = 0
        instr = []   # (byte offset, region key or None = cold, issue weight)
        for i, x in enumerate(body):
            if i in cold:
                instr.append((x["addr"], None, 1))
                continue
            r = final[i]
            if r is None:
                unmapped += 1
                r = ("UNMAPPED", True)
            if r[0] != "ENTRY" and loops and not any(a <= i <= b for a, b in loops):
                r = ("ENTRY", True)   # loop preheader / exit copy: runs once per warp
            key = r[0] + (":full" if r[1] else "")
            n = 1
            cm = re.search(r"CALL\.\w+(?:\.NOINC)?\s+`\((\S+?)\)", x["text"])
            if cm and cm.group(1) in sub_size and not x["text"].startswith("@"):
                n += sub_size[cm.group(1)]
            reg[key] = reg.get(key, 0) + n
            instr.append((x["addr"], key, n))
        out[name] = dict(regions=reg, unmapped=unmapped, total=sum(reg.values()), instr=instr)
    return out


if __name__ == "__main__":
    res = kernel_costs(sys.argv[1] if len(sys.argv) > 1 else ".*")
    for v in res.values():
        v.pop("instr")
    print(json.dumps(res, indent=1))
