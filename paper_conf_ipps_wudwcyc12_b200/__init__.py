"""B200-native fused relational-operator hot path (Wu et al., IPDPSW 2012).

The product is ``libra.so`` (C ABI in ``include/ra.h``): hand-written sm_100a
kernels for the fused SELECT chain, fused TPC-H Q1 and the kernel-fission
pipeline.  This package is the thin Python layer above it:

* ``ra_*`` — one-to-one ctypes bindings of the C entry points (``_ra.py``);
* ``select_chain``, ``q1``, ``q1_finalize``, ``fission_run``,
  ``q1_fission_run``, ``q1_encode``, ``q1_narrow``, ``q1_narrow_fission_run``,
  ``select_rows`` — conveniences
  that take torch tensors, allocate outputs/workspaces with torch (device
  memory and streams are PyTorch's; nothing else is) and call the bindings.

There is no CPU or PyTorch fallback: every step of the path runs in libra.so.
"""
from __future__ import annotations

import ctypes

from ._ra import *  # noqa: F401,F403
from ._ra import (RA_E_CAPACITY, RA_E_DOMAIN, RA_OK, RA_Q1_GROUPS, make_preds, ra_fission_run,
                  ra_fission_workspace_bytes, ra_lineitem, ra_q1, ra_q1_finalize, ra_q1_partial,
                  ra_q1_fission_run, ra_q1_fission_workspace_bytes, ra_q1_row, ra_q1_workspace_bytes,
                  ra_select_chain, ra_select_workspace_bytes, ra_lineitem_narrow, ra_lineitem_narrow_out,
                  ra_q1_encode, ra_q1_narrow, ra_q1_narrow_fission_run, ra_q1_narrow_fission_workspace_bytes,
                  ra_payload, ra_select_rows, ra_select_rows_workspace_bytes, ra_select_multi, RA_MAX_PREDS,
                  ra_select_multi_workspace_bytes)

Q1_CUTOFF_DELTA90 = 10471  # 1998-12-01 - 90 days = 1998-09-02
LINEITEM_COLUMNS = ("shipdate", "returnflag", "linestatus", "quantity", "extendedprice", "discount", "tax")
# narrow (f4) encoding: column -> torch dtype name (ra.h ra_lineitem_narrow)
NARROW_COLUMNS = (("shipdate", "uint16"), ("group", "uint8"), ("quantity", "uint16"), ("discount", "uint8"),
                  ("tax", "uint8"), ("extendedprice", "uint32"))

_WS: dict = {}


def _torch():
    import torch
    return torch


def _stream_handle(stream) -> int:
    torch = _torch()
    if stream is None:
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream) if hasattr(stream, "cuda_stream") else int(stream)


def _used_on(stream, *tensors):
    """Tensors allocated here (on the current stream) but written by kernels
    enqueued on ``stream``: record that use with the caching allocator, so
    their memory is not handed out again before ``stream``'s work completes."""
    torch = _torch()
    if stream is None:
        return
    for t in tensors:
        if t is None:
            continue
        s = stream if isinstance(stream, torch.cuda.Stream) else \
            torch.cuda.ExternalStream(int(stream), device=t.device)
        if s != torch.cuda.current_stream(t.device):
            t.record_stream(s)


def workspace(device, kind: str, nbytes: int, stream=None):
    """Zero-initialised workspace tensor, cached per (device, kind, stream).

    One ``kind`` per entry point (ra.h: a workspace handed to another entry
    point must be re-initialised).  The zero fill runs on the current stream
    and is complete before this returns: the kernels, and the fission runtimes'
    own streams, may use the workspace from any stream.  A replaced (smaller)
    workspace was recorded on the stream that used it, so the allocator keeps
    its memory until that stream's work is done."""
    torch = _torch()
    key = (str(device), kind, _stream_handle(stream))
    ws = _WS.get(key)
    if ws is None or ws.numel() < nbytes:
        if torch.cuda.is_current_stream_capturing():
            raise RuntimeError(f"workspace {kind!r} for this stream must be created before CUDA-graph capture "
                               "(make one call on the capture stream first)")
        ws = torch.zeros(max(256, nbytes), dtype=torch.uint8, device=device)
        # Root cause of round 1's one-off Q1-fission mismatch: without this the
        # fill kernel (current stream) could still be running while the fission
        # streams (not ordered after it) had already accumulated chunk partials
        # into the same bytes, zeroing part of the result.
        torch.cuda.current_stream(device).synchronize()
        _used_on(stream, ws)
        _WS[key] = ws
    return ws


def select_chain(x, preds, fused: bool = True, out=None, count=None, stream=None):
    """Fused (or unfused) SELECT chain over a CUDA int32 tensor.

    Returns ``(out, count)``: ``out[:count]`` holds the selected values in
    input order; ``count`` is a 1-element int64 CUDA tensor (not synchronised).
    """
    torch = _torch()
    if not (x.is_cuda and x.dtype == torch.int32 and x.is_contiguous()):
        raise ValueError("x must be a contiguous CUDA int32 tensor")
    n, k = x.numel(), len(preds)
    if out is None:
        out = torch.empty(max(1, n), dtype=torch.int32, device=x.device)
    if count is None:
        count = torch.empty(1, dtype=torch.int64, device=x.device)
    _used_on(stream, out, count)
    need = ra_select_workspace_bytes(n, k, int(fused))
    ws = workspace(x.device, "select_fused" if fused else "select_unfused", need, stream)
    P = make_preds(preds)
    ra_select_chain(x.data_ptr(), n, P, k, int(fused), out.data_ptr(), out.numel(), count.data_ptr(),
                    ws.data_ptr(), ws.numel(), _stream_handle(stream))
    return out, count


def select_multi(x, chains, outs=None, stream=None):
    """Several SELECTs on the same CUDA int32 tensor in one pass (Fig 2(c)).

    ``chains``: list of 1..RA_MAX_OUTPUTS predicate chains.  Returns
    ``(outs, counts)``: ``outs[o][:counts[o]]`` is chain o's selection in
    input order; ``counts`` a CUDA int64 tensor (not synchronised)."""
    torch = _torch()
    if not (x.is_cuda and x.dtype == torch.int32 and x.is_contiguous()):
        raise ValueError("x must be a contiguous CUDA int32 tensor")
    n, M = x.numel(), len(chains)
    if outs is None:
        outs = [torch.empty(max(1, n), dtype=torch.int32, device=x.device) for _ in range(M)]
    counts = torch.empty(max(1, M), dtype=torch.int64, device=x.device)
    keep = [make_preds(c) for c in chains]
    ch = (ctypes.c_void_p * M)(*[ctypes.addressof(p) for p in keep])
    ks = (ctypes.c_int * M)(*[len(c) for c in chains])
    op = (ctypes.c_void_p * M)(*[o.data_ptr() for o in outs])
    caps = (ctypes.c_int64 * M)(*[o.numel() for o in outs])
    cp = (ctypes.c_void_p * M)(*[counts.data_ptr() + 8 * o for o in range(M)])
    _used_on(stream, counts, *outs)
    ws = workspace(x.device, "select_multi", ra_select_multi_workspace_bytes(n), stream)
    ra_select_multi(x.data_ptr(), n, ch, ks, M, op, caps, cp, ws.data_ptr(), ws.numel(), _stream_handle(stream))
    return outs, counts


def select_rows(key, preds, payloads=(), rowids: bool = True, out_cap=None, stream=None):
    """Tuple SELECT (Table I) over a CUDA int32 key column and payload columns
    (CUDA 4- or 8-byte tensors of the same length), one fused pass.

    Returns ``(rowids, outs, count)``: ``rowids[:count]`` (uint32, or None),
    ``outs[j][:count]`` the payload fields of the selected rows in input order,
    ``count`` a 1-element int64 CUDA tensor (not synchronised)."""
    torch = _torch()
    if not (key.is_cuda and key.dtype == torch.int32 and key.is_contiguous()):
        raise ValueError("key must be a contiguous CUDA int32 tensor")
    n, k = key.numel(), len(preds)
    cap = n if out_cap is None else int(out_cap)
    ids = torch.empty(max(1, cap), dtype=torch.uint32, device=key.device) if rowids else None
    outs, pl = [], (ra_payload * max(1, len(payloads)))()
    for j, c in enumerate(payloads):
        if not (c.is_cuda and c.is_contiguous() and c.numel() == n and c.element_size() in (4, 8)):
            raise ValueError("payloads must be contiguous CUDA 4/8-byte tensors of the key's length")
        o = torch.empty(max(1, cap), dtype=c.dtype, device=key.device)
        outs.append(o)
        pl[j].col, pl[j].out, pl[j].elem_bytes = c.data_ptr(), o.data_ptr(), c.element_size()
    count = torch.empty(1, dtype=torch.int64, device=key.device)
    _used_on(stream, ids, count, *outs)
    need = ra_select_rows_workspace_bytes(n, k)
    ws = workspace(key.device, "select_rows", need, stream)
    P = make_preds(preds)
    ra_select_rows(key.data_ptr(), n, P, k, ids.data_ptr() if ids is not None else 0, pl, len(payloads), cap,
                   count.data_ptr(), ws.data_ptr(), ws.numel(), _stream_handle(stream))
    return ids, outs, count


def lineitem_struct(cols) -> ra_lineitem:
    return ra_lineitem(*[cols[name].data_ptr() for name in LINEITEM_COLUMNS])


def q1(cols, cutoff: int = Q1_CUTOFF_DELTA90, partial=None, stream=None):
    """Fused Q1 over CUDA lineitem columns; returns the device partial (uint8[400])."""
    torch = _torch()
    sd = cols["shipdate"]
    n = sd.numel()
    if partial is None:
        partial = torch.empty(ctypes.sizeof(ra_q1_partial), dtype=torch.uint8, device=sd.device)
        _used_on(stream, partial)
    ws = workspace(sd.device, "q1", ra_q1_workspace_bytes(n), stream)
    ra_q1(lineitem_struct(cols), n, int(cutoff), partial.data_ptr(), ws.data_ptr(), ws.numel(),
          _stream_handle(stream))
    return partial


def narrow_empty(n: int, device):
    """Device tensors for an n-row narrow lineitem (16-B aligned torch allocations)."""
    torch = _torch()
    return {name: torch.empty(max(1, n), dtype=getattr(torch, dt), device=device)[:n] for name, dt in NARROW_COLUMNS}


def q1_encode(cols, out=None, stream=None):
    """Re-encode wide CUDA lineitem columns into the narrow layout (f4).

    Returns ``(narrow_cols, status)``; ``status`` is a 1-element uint32 CUDA
    tensor (0 = exact re-encoding; bits as in ra.h), not synchronised."""
    torch = _torch()
    sd = cols["shipdate"]
    n = sd.numel()
    if out is None:
        out = narrow_empty(n, sd.device)
    status = torch.empty(1, dtype=torch.uint32, device=sd.device)
    _used_on(stream, status, *out.values())
    h_out = ra_lineitem_narrow_out(*[out[name].data_ptr() for name, _ in NARROW_COLUMNS])
    ra_q1_encode(lineitem_struct(cols), n, h_out, status.data_ptr(), _stream_handle(stream))
    return out, status


def q1_narrow(ncols, cutoff: int = Q1_CUTOFF_DELTA90, partial=None, stream=None):
    """Fused Q1 over narrow CUDA columns; returns the device partial (uint8[400])."""
    torch = _torch()
    sd = ncols["shipdate"]
    n = sd.numel()
    if partial is None:
        partial = torch.empty(ctypes.sizeof(ra_q1_partial), dtype=torch.uint8, device=sd.device)
        _used_on(stream, partial)
    ws = workspace(sd.device, "q1", ra_q1_workspace_bytes(n), stream)
    h = ra_lineitem_narrow(*[ncols[name].data_ptr() for name, _ in NARROW_COLUMNS])
    ra_q1_narrow(h, n, int(cutoff), partial.data_ptr(), ws.data_ptr(), ws.numel(), _stream_handle(stream))
    return partial


def partials_from_bytes(buf: bytes, n_partials: int = 1):
    arr = (ra_q1_partial * n_partials)()
    ctypes.memmove(arr, buf, ctypes.sizeof(arr))
    return arr


def q1_finalize(partials):
    """Host finalize of one or more partials (ctypes array or bytes).

    Returns ``(rows, rc)`` with rows as dicts (exact ints, AVG doubles) and
    ``rc`` = RA_OK or RA_E_DOMAIN.
    """
    if isinstance(partials, (bytes, bytearray)):
        partials = partials_from_bytes(bytes(partials), len(partials) // ctypes.sizeof(ra_q1_partial))
    rows = (ra_q1_row * RA_Q1_GROUPS)()
    nrows = ctypes.c_int(0)
    rc = ra_q1_finalize(partials, len(partials), rows, ctypes.byref(nrows))
    out = []
    for r in rows[:nrows.value]:
        out.append({
            "returnflag": chr(r.returnflag), "linestatus": chr(r.linestatus),
            "count_order": r.count_order, "sum_qty": r.sum_qty, "sum_base_price": r.sum_base_price,
            "sum_disc_price": (r.sum_disc_price_hi << 64) | r.sum_disc_price_lo,
            "sum_charge": (r.sum_charge_hi << 64) | r.sum_charge_lo, "sum_disc": r.sum_disc,
            "avg_qty": r.avg_qty, "avg_price": r.avg_price, "avg_disc": r.avg_disc,
        })
    return out, rc


def fission_run(h_in, preds, chunk_rows: int, streams, fused: bool = True, h_out=None,
                h_chunk_counts=None, device=None):
    """Host-resident SELECT chain with kernel fission (synchronous).

    ``h_in``: pinned CPU int32 tensor.  Returns ``(h_out, count)`` with
    ``h_out[:count]`` the selected values.
    """
    torch = _torch()
    if not (h_in.dtype == torch.int32 and h_in.is_contiguous() and (h_in.numel() == 0 or h_in.is_pinned())):
        raise ValueError("h_in must be a pinned contiguous int32 CPU tensor")
    n, k = h_in.numel(), len(preds)
    chunk_rows = max(1, min(int(chunk_rows), max(1, n)))
    nchunks = (n + chunk_rows - 1) // chunk_rows
    device = device or torch.device("cuda", torch.cuda.current_device())
    if h_out is None:
        h_out = torch.empty(max(1, n), dtype=torch.int32, pin_memory=True)
    if h_chunk_counts is None or h_chunk_counts.numel() < max(1, nchunks):
        h_chunk_counts = torch.zeros(max(1, nchunks), dtype=torch.int64, pin_memory=True)
    S = len(streams)
    sarr = (ctypes.c_void_p * S)(*[_stream_handle(s) for s in streams])
    ws = workspace(device, f"fission_{int(fused)}_{S}", ra_fission_workspace_bytes(chunk_rows, S, k, int(fused)))
    P = make_preds(preds)
    cnt = ctypes.c_int64(0)
    ra_fission_run(h_in.data_ptr(), n, P, k, int(fused), chunk_rows, sarr, S, h_out.data_ptr(),
                   h_out.numel(), ctypes.byref(cnt), h_chunk_counts.data_ptr(), ws.data_ptr(),
                   ws.numel())
    return h_out, int(cnt.value)


def q1_fission_run(h_cols, chunk_rows: int, streams, cutoff: int = Q1_CUTOFF_DELTA90, device=None):
    """Host-resident Q1 under kernel fission (synchronous).

    ``h_cols``: dict of pinned contiguous CPU tensors (LINEITEM_COLUMNS).
    Returns the whole query's ``ra_q1_partial`` (pass it to ``q1_finalize``).
    """
    torch = _torch()
    n = h_cols["shipdate"].numel()
    for name in LINEITEM_COLUMNS:
        t = h_cols[name]
        if t.numel() != n or t.device.type != "cpu" or not t.is_contiguous() or (n and not t.is_pinned()):
            raise ValueError(f"h_cols[{name!r}] must be a pinned contiguous CPU tensor of {n} rows")
    chunk_rows = max(1, min(int(chunk_rows), max(1, n)))
    device = device or torch.device("cuda", torch.cuda.current_device())
    S = len(streams)
    sarr = (ctypes.c_void_p * S)(*[_stream_handle(s) for s in streams])
    ws = workspace(device, f"q1_fission_{S}", ra_q1_fission_workspace_bytes(chunk_rows, S))
    part = ra_q1_partial()
    ra_q1_fission_run(lineitem_struct(h_cols), n, int(cutoff), chunk_rows, sarr, S, part, ws.data_ptr(),
                      ws.numel())
    return part


def q1_narrow_fission_run(h_cols, chunk_rows: int, streams, cutoff: int = Q1_CUTOFF_DELTA90, device=None):
    """Host-resident narrow Q1 under kernel fission (synchronous, f1 x f4).

    ``h_cols``: dict of pinned contiguous CPU tensors (NARROW_COLUMNS).
    Returns the whole query's ``ra_q1_partial``.
    """
    torch = _torch()
    n = h_cols["shipdate"].numel()
    for name, _ in NARROW_COLUMNS:
        t = h_cols[name]
        if t.numel() != n or t.device.type != "cpu" or not t.is_contiguous() or (n and not t.is_pinned()):
            raise ValueError(f"h_cols[{name!r}] must be a pinned contiguous CPU tensor of {n} rows")
    chunk_rows = max(1, min(int(chunk_rows), max(1, n)))
    device = device or torch.device("cuda", torch.cuda.current_device())
    S = len(streams)
    sarr = (ctypes.c_void_p * S)(*[_stream_handle(s) for s in streams])
    ws = workspace(device, f"q1n_fission_{S}", ra_q1_narrow_fission_workspace_bytes(chunk_rows, S))
    part = ra_q1_partial()
    h = ra_lineitem_narrow(*[h_cols[name].data_ptr() for name, _ in NARROW_COLUMNS])
    ra_q1_narrow_fission_run(h, n, int(cutoff), chunk_rows, sarr, S, part, ws.data_ptr(), ws.numel())
    return part
