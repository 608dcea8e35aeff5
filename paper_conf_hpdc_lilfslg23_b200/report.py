"""Host-side reports over fetched table entries.

Renders the entries the way the paper's tool reports them:

* detector lines, ``#GPU-FPX LOC-EXCEP INFO: in kernel [K], NaN found @ L [FP32]``
  (Listing 6), one per (site, kind, fmt) with a destination-only
  (flow NONE) entry;
* analyzer lines, ``#GPU-FPX-ANA <STATE>: ...`` with the Table 2 state
  (Appearance / Propagation / Disappearance) of FLOW entries;
* the Table-4 summary: distinct sites per (format, kind).

Pure formatting of integers already computed by the device table; no
classification happens here.
"""
from __future__ import annotations

import numpy as np

FMT_NAMES = {0: "FP32", 1: "FP64", 2: "FP16", 3: "BF16"}
KIND_NAMES = {0: "NaN", 1: "INF", 2: "SUB", 3: "DIV0"}
STATE_NAMES = {1: "APPEARANCE", 2: "PROPAGATION", 3: "DISAPPEARANCE"}  # Table 2 (GEN / PROP / KILL)


def _site_label(site: int, names: dict | None):
    """(kernel, location) of a site; names maps site -> (kernel, location) or kernel."""
    if names and site in names:
        v = names[site]
        if isinstance(v, tuple):
            return v[0], v[1]
        return str(v), "/unknown_path"
    return f"site_{site:#010x}", "/unknown_path"


def detector_lines(entries: np.ndarray, names: dict | None = None) -> list[str]:
    """One line per destination-only entry, in key order."""
    out = []
    for e in entries:
        if int(e["flow"]) != 0:
            continue
        kernel, loc = _site_label(int(e["site"]), names)
        out.append(
            f"#GPU-FPX LOC-EXCEP INFO: in kernel [{kernel}], {KIND_NAMES[int(e['kind'])]} found @ {loc} "
            f"in [{kernel}]:{int(e['site']) & 0xFFFF} [{FMT_NAMES[int(e['fmt'])]}] "
            f"count={int(e['count'])} first={int(e['first_index'])}"
        )
    return out


def analyzer_lines(entries: np.ndarray, names: dict | None = None) -> list[str]:
    """One line per FLOW entry: the Table 2 state of the instruction site; with
    FPX_MODE_FLOW_DETAIL entries also the Comparison state and the source
    operand that carried the exceptional value (fn4 P:99)."""
    out = []
    for e in entries:
        flow = int(e["flow"])
        if flow == 0:
            continue
        kernel, loc = _site_label(int(e["site"]), names)
        det = int(e["detail"]) if "detail" in e.dtype.names else 0
        state = "COMPARISON/" + STATE_NAMES[flow] if det & 4 else STATE_NAMES[flow]
        src = f" from source {(det & 3) - 1}" if det & 3 else ""
        out.append(
            f"#GPU-FPX-ANA {state}: {KIND_NAMES[int(e['kind'])]}{src} @ {loc} in [{kernel}]:"
            f"{int(e['site']) & 0xFFFF} [{FMT_NAMES[int(e['fmt'])]}] count={int(e['count'])} "
            f"first={int(e['first_index'])}"
        )
    return out


def t4_table(entries: np.ndarray) -> dict:
    """{(fmt, kind): number of distinct sites} — the Table 4 metric."""
    out = {}
    for fmt in FMT_NAMES:
        for kind in KIND_NAMES:
            sel = entries[(entries["fmt"] == fmt) & (entries["kind"] == kind)]
            if len(sel):
                out[(fmt, kind)] = int(len(np.unique(sel["site"])))
    return out


def t4_lines(entries: np.ndarray) -> list[str]:
    """Table 4 layout: per format, distinct sites with NaN / INF / SUB / DIV0."""
    t = t4_table(entries)
    lines = ["fmt    NAN   INF   SUB  DIV0"]
    for fmt, fname in FMT_NAMES.items():
        row = [t.get((fmt, k), 0) for k in range(4)]
        if any(row):
            lines.append(f"{fname:5s} " + " ".join(f"{v:5d}" for v in row))
    return lines
