"""Tiny DSL for the paper's racy / fixed listings (tests/golden/listings.txt) → tracegen Program.

Each access-producing call may carry a label ``@L``; the accesses it produces are named
``L`` (single access), ``L.i`` (kernel argument i), ``L.w`` / ``L.r`` (memcpy destination / source).
"""
from __future__ import annotations

import os
from dataclasses import dataclass, field

from tracegen.program import (CPY_D2D, CPY_D2H, CPY_H2D, CPY_H2H, MEM_DEVICE, MEM_MANAGED, MEM_PAGEABLE,
                              MEM_PINNED, MODE_R, MODE_RW, MODE_W, Program)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "listings.txt")
KINDS = dict(device=MEM_DEVICE, managed=MEM_MANAGED, pinned=MEM_PINNED, pageable=MEM_PAGEABLE)
CPY = dict(h2h=CPY_H2H, h2d=CPY_H2D, d2h=CPY_D2H, d2d=CPY_D2D)
MODES = dict(R=MODE_R, W=MODE_W, RW=MODE_RW)


@dataclass
class Listing:
    name: str
    program: Program
    op_access_labels: dict = field(default_factory=dict)   # op index -> [label per access]
    expect: list = field(default_factory=list)             # [(earlier, later, granules|None)]


def _split_label(tokens):
    label = None
    out = []
    for t in tokens:
        if "@" in t:
            t, label = t.split("@", 1)
            if not t:
                continue
        out.append(t)
    return out, label


def parse(path: str = GOLDEN) -> list[Listing]:
    listings: list[Listing] = []
    cur = None
    env: dict = {}
    for raw in open(path):
        line = raw.split("#", 1)[0].strip()
        if not line:
            continue
        tok, label = _split_label(line.split())
        cmd, rest = tok[0], tok[1:]
        if cmd == "listing":
            cur = Listing(rest[0], Program())
            listings.append(cur)
            env = {"default": 0, "legacy": 1, "ptds": 2}   # CUDA's stream handles
            continue
        p = cur.program

        def ptr(t):
            if "+" in t:
                v, off = t.split("+")
                return env[v] + int(off)
            return env[t]

        k = len(p.ops)
        labels = None
        if cmd == "malloc":
            env[rest[0]] = p.malloc(int(rest[1]), KINDS[rest[2]] if len(rest) > 2 else MEM_DEVICE)
        elif cmd == "stream":
            env[rest[0]] = p.stream_create(nonblocking=len(rest) > 1 and rest[1] == "nonblocking")
        elif cmd == "kernel":
            args = []
            for a in rest[1:]:
                v, m = a.split(":")
                args.append((ptr(v), MODES[m]))
            p.kernel(env[rest[0]], args)
            if label:
                labels = [label] if len(args) == 1 else [f"{label}.{i}" for i in range(len(args))]
        elif cmd == "ssync":
            p.stream_sync(env[rest[0]])
        elif cmd == "dsync":
            p.device_sync()
        elif cmd == "erecord":
            env.setdefault(rest[0], p.new_event())
            p.event_record(env[rest[0]], env[rest[1]])
        elif cmd == "esync":
            p.event_sync(env[rest[0]])
        elif cmd == "swait":
            p.stream_wait_event(env[rest[0]], env[rest[1]])
        elif cmd == "squery":
            p.stream_query(env[rest[0]], rest[1] == "ok")
        elif cmd == "memcpy":
            p.memcpy(ptr(rest[0]), ptr(rest[1]), int(rest[2]), CPY[rest[3]])
            labels = [f"{label}.w", f"{label}.r"] if label else None
        elif cmd == "memcpya":                         # cudaMemcpyAsync(dst, src, n, kind, stream)
            p.memcpy_async(ptr(rest[0]), ptr(rest[1]), int(rest[2]), CPY[rest[3]], env[rest[4]])
            labels = [f"{label}.w", f"{label}.r"] if label else None
        elif cmd == "memset":
            if len(rest) > 2:
                p.memset_async(ptr(rest[0]), int(rest[1]), env[rest[2]])
            else:
                p.memset(ptr(rest[0]), int(rest[1]))
            labels = [label] if label else None
        elif cmd == "host":
            p.host_access(ptr(rest[0]), int(rest[1]), 1 if rest[2] == "W" else 0)
            labels = [label] if label else None
        elif cmd in ("isend", "irecv"):
            r = (p.isend if cmd == "isend" else p.irecv)(ptr(rest[1]), int(rest[2]))
            env[rest[0]] = r
            labels = [label] if label else None
        elif cmd == "wait":
            p.wait(env[rest[0]])
        elif cmd == "test":
            p.test(env[rest[0]], rest[1] == "ok")
        elif cmd in ("send", "recv"):
            (p.send if cmd == "send" else p.recv)(ptr(rest[0]), int(rest[1]))
            labels = [label] if label else None
        elif cmd == "free":
            p.free(env[rest[0]])
        elif cmd == "mode":
            p.default_stream_mode(rest[0] == "per-thread")
        elif cmd == "thread":
            p.set_thread(int(rest[0]))
        elif cmd == "tcreate":
            p.thread_create(int(rest[0]))
        elif cmd == "tjoin":
            p.thread_join(int(rest[0]))
        elif cmd == "expect":
            if rest[0] == "race":
                cur.expect.append((rest[1], rest[2], int(rest[3]) if len(rest) > 3 else None))
            continue
        else:
            raise ValueError(f"unknown listing command {cmd}")
        if labels:
            cur.op_access_labels[k] = labels
    return listings


def label_events(listing: Listing, events, op_first_event: list[int]) -> dict[int, str]:
    """Map ACCESS event ids to labels, given the first event id each op lowered to."""
    out = {}
    n = len(events)
    for k, labels in listing.op_access_labels.items():
        lo = op_first_event[k]
        hi = op_first_event[k + 1] if k + 1 < len(op_first_event) else n
        acc = [i for i in range(lo, hi) if int(events[i]["kind"]) == 0]
        for i, lab in zip(acc, labels):
            out[i] = lab
    return out


def observed_pairs(runs, ev_labels: dict[int, str]) -> dict[tuple[str, str], int]:
    out: dict = {}
    for r in runs:
        key = (ev_labels.get(int(r["earlier"]), f"#{int(r['earlier'])}"),
               ev_labels.get(int(r["later"]), f"#{int(r['later'])}"))
        out[key] = out.get(key, 0) + int(r["g_end"] - r["g_begin"])
    return out
