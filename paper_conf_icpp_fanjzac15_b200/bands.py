"""Row-band sharding of ONE image over the ranks of a process group
(DESIGN.md sec. 9).

One process per GPU.  Rank g owns output rows [row0, row1) (multiples of 4,
so no 4x4 downscale block of PAPER.md L130 straddles two bands).  The method
couples the bands in exactly two places:

* halo rows: the upscale of rows row0..row1-1 reads D rows row0/4-1 .. row1/4
  (L146) and the Sobel / 3x3 overshoot window one row (L158-L172, L182), so a
  band's input buffer holds 4 extra image rows above and below
  (`halo_rows`, the C ABI's sharp_band_halo); `exchange_halos` fetches them
  from the neighbouring ranks (point-to-point send/recv; NCCL over NVLink on
  GPUs, gloo on CPU);
* the pEdge mean (L174): each rank sums pEdge over its own rows
  (sharp_band_edge_sum), one all-reduce of a 64-bit integer adds the partials,
  and every rank builds the identical LUTs from the identical S
  (sharp_band_sharpen) -- so the bands are bit-identical to the same rows of
  the whole-image result.

torch.distributed is plumbing only (the collective and the P2P transfers);
every pixel is computed by libsharp.so.
"""
import torch
import torch.distributed as dist

HALO = 4  # image rows of halo per side


def band_rows(h, world, rank):
    """Rows [row0, row1) of rank `rank`: the h/4 downscale block rows split
    as evenly as possible (the first (h/4) % world ranks get one more)."""
    if h % 4 or h < 8 or world < 1 or not 0 <= rank < world:
        raise ValueError("bad band request")
    blocks = h // 4
    if blocks < world:
        raise ValueError(f"{h} rows cannot feed {world} bands of >= 4 rows")
    base, rem = divmod(blocks, world)
    start = rank * base + min(rank, rem)
    count = base + (1 if rank < rem else 0)
    return 4 * start, 4 * (start + count)


def halo_rows(h, row0, row1):
    """Image rows [in0, in1) a band's input buffer holds (sharp_band_halo)."""
    return max(row0 - HALO, 0), min(row1 + HALO, h)


def _world(group):
    if not (dist.is_available() and dist.is_initialized()):
        return 1, 0
    return dist.get_world_size(group), dist.get_rank(group)


def exchange_halos(own, h, row0, row1, group=None):
    """own: this rank's rows [row0, row1) ([rows, w] uint8, any device).
    Returns the band buffer of rows [in0, in1): own plus up to HALO rows from
    each neighbour (rank-1 above, rank+1 below), by point-to-point transfers.
    Every rank must call it (it pairs sends with the neighbours' receives)."""
    world, rank = _world(group)
    in0, in1 = halo_rows(h, row0, row1)
    rows, w = own.shape
    if rows != row1 - row0:
        raise ValueError("own rows do not match [row0, row1)")
    band = torch.empty((in1 - in0, w), dtype=own.dtype, device=own.device)
    top, bot = row0 - in0, in1 - row1
    band[top:top + rows].copy_(own)
    if world == 1:
        if top or bot:
            raise ValueError("a single rank must own the whole image")
        return band
    ops = []
    # gloo moves host tensors only (a CUDA band under gloo -- the one-GPU
    # test hook -- is staged through host copies); NCCL moves device memory
    host = own.is_cuda and dist.get_backend(group) == "gloo"
    stage = (lambda t: t.cpu()) if host else (lambda t: t)
    up_recv = stage(band[:top]) if top else None
    dn_recv = stage(band[top + rows:]) if bot else None
    peer = (lambda r: dist.get_global_rank(group, r)) if group is not None else (lambda r: r)
    if rank > 0:  # exchange with the band above: it needs our first rows, we need its last
        ops.append(dist.P2POp(dist.isend, stage(own[:HALO].contiguous()), peer(rank - 1), group))
        ops.append(dist.P2POp(dist.irecv, up_recv, peer(rank - 1), group))
    if rank < world - 1:
        ops.append(dist.P2POp(dist.isend, stage(own[rows - HALO:].contiguous()), peer(rank + 1), group))
        ops.append(dist.P2POp(dist.irecv, dn_recv, peer(rank + 1), group))
    for req in dist.batch_isend_irecv(ops):
        req.wait()
    if host:
        if top:
            band[:top].copy_(up_recv)
        if bot:
            band[top + rows:].copy_(dn_recv)
    return band


def sharpen_band(sharpener, band, w, h, row0, row1, params=None, out=None, group=None):
    """Sharpen this rank's rows [row0, row1) of a w x h image.

    band: CUDA uint8 tensor of image rows halo_rows(h, row0, row1).
    Runs sharp_band_edge_sum -> all-reduce(sum) of the u64 partial over the
    group (skipped when not distributed) -> sharp_band_sharpen, all on the
    current CUDA stream.  Returns (out, S): out = [row1-row0, w] uint8 and S
    the image's pEdge sum (a 1-element int64 CUDA tensor)."""
    if out is None:
        out = torch.empty((row1 - row0, w), dtype=torch.uint8, device=band.device)
    stream = torch.cuda.current_stream(band.device)
    sharpener.set_stream(stream)
    s = torch.zeros(1, dtype=torch.int64, device=band.device)  # u64 bits; S < 2^40
    sharpener.band_edge_sum(band, w, h, row0, row1, s)
    world, _ = _world(group)
    if world > 1:  # the L174 reduction across bands (host-staged under gloo)
        if s.is_cuda and dist.get_backend(group) == "gloo":
            t = s.cpu()
            dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
            s.copy_(t)
        else:
            dist.all_reduce(s, op=dist.ReduceOp.SUM, group=group)
    sharpener.band_sharpen(band, w, h, row0, row1, s, out, params)
    return out, s


# ---------------------------------------------------------------------------
# Fused peer-memory exchange:
# the halo rows and the u64 pEdge partials move by direct stores into the
# neighbours' / every rank's window (NVLink peer mappings via CUDA IPC) with
# epoch flags -- libsharp.so's sharp_band_p2p_halo / sharp_band_p2p_allreduce
# -- instead of NCCL send/recv + all-reduce.  torch.distributed only carries
# the one-time exchange of the IPC handles.

def _device_view(addr, nbytes, device):
    """A torch uint8 tensor aliasing device memory [addr, addr + nbytes)."""
    class _Mem:
        __cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (addr, False), "version": 3}
    return torch.as_tensor(_Mem(), device=device)


class P2PBand:
    """This rank's band of a w x h image and its exchange window.

    Multi-process (one GPU per rank): P2PBand(sharpener, w, h, group) --
    windows are exchanged once as CUDA IPC handles over `group`.
    Single-process (tests, several bands on one device): pass `windows`, the
    list of every band's window address, and `rank`.
    Use: write this band's rows into `own` ([rows, w] uint8 view), then
    step(epoch, out, params) with epochs 1, 2, 3, ... (the same on every rank)."""

    def __init__(self, sharpener, w, h, group=None, rank=None, world=None, window=None, windows=None):
        from . import binding as B
        self.B, self.sh, self.w, self.h = B, sharpener, w, h
        if world is None:
            world, rank = _world(group)
        self.world, self.rank = world, rank
        self.rows = [band_rows(h, world, g) for g in range(world)]
        self.row0, self.row1 = self.rows[rank]
        self.rows_own = self.row1 - self.row0
        if w % 16 or self.rows_own < HALO:
            raise ValueError("P2P bands need w % 16 == 0 and >= 4 rows per band")
        self.nbytes = B.sharp_p2p_window_bytes(w, self.rows_own)
        self._owned = window is None
        self.window = window if window is not None else B.sharp_p2p_window_create(w, self.rows_own)
        self._opened = []
        if windows is None:  # multi-process: exchange IPC handles once
            if world > 1:
                handles = [None] * world
                dist.all_gather_object(handles, B.sharp_ipc_get_handle(self.window), group=group)
                windows = []
                for g, hnd in enumerate(handles):
                    if g == rank:
                        windows.append(self.window)
                    else:
                        p = B.sharp_ipc_open_handle(hnd)
                        self._opened.append(p)
                        windows.append(p)
            else:
                windows = [self.window]
        self.windows = list(windows)
        dev = torch.device("cuda", torch.cuda.current_device())
        base = self.window + B.SHARP_P2P_CTL_BYTES
        self.own = _device_view(base + HALO * w, self.rows_own * w, dev).view(self.rows_own, w)
        in0, in1 = halo_rows(h, self.row0, self.row1)
        first = base + (in0 - (self.row0 - HALO)) * w
        self.band = _device_view(first, (in1 - in0) * w, dev).view(in1 - in0, w)
        self.partial = torch.zeros(1, dtype=torch.int64, device=dev)
        self.total = torch.zeros(1, dtype=torch.int64, device=dev)

    def step(self, epoch, out, params=None):
        """Halo push + pass 1 + peer all-reduce + pass 2 of image `epoch`, on
        the sharpener's stream.  out: [rows, w] uint8 CUDA tensor."""
        B, g = self.B, self.rank
        up = self.windows[g - 1] if g > 0 else None
        dn = self.windows[g + 1] if g < self.world - 1 else None
        up_rows = self.rows[g - 1][1] - self.rows[g - 1][0] if g > 0 else 0
        B.sharp_band_p2p_halo(self.sh.ctx, self.window, self.w, self.rows_own, up, up_rows, dn, epoch)
        self.sh.band_edge_sum(self.band, self.w, self.h, self.row0, self.row1, self.partial)
        B.sharp_band_p2p_allreduce(self.sh.ctx, self.windows, g, self.partial, epoch, self.total)
        self.sh.band_sharpen(self.band, self.w, self.h, self.row0, self.row1, self.total, out, params)
        return out

    def step_fused(self, epoch, out, params=None, grid_cap=0):
        """Halo push, then pass 1 + the peer-memory all-reduce + pass 2 in ONE
        step-kernel launch (sharp_band_p2p_sharpen).  grid_cap: CTAs of the
        persistent grid (bands sharing one GPU must co-reside)."""
        B, g = self.B, self.rank
        up = self.windows[g - 1] if g > 0 else None
        dn = self.windows[g + 1] if g < self.world - 1 else None
        up_rows = self.rows[g - 1][1] - self.rows[g - 1][0] if g > 0 else 0
        B.sharp_band_p2p_halo(self.sh.ctx, self.window, self.w, self.rows_own, up, up_rows, dn, epoch)
        B.sharp_band_p2p_sharpen(self.sh.ctx, self.windows, g, self.w, self.h, self.row0, self.row1, epoch, params,
                                 out, grid_cap)
        return out

    def step_one_launch(self, epoch, out, params=None, grid_cap=0):
        """Halo push + pass 1 + the peer-memory all-reduce + pass 2 in ONE
        step-kernel launch (sharp_band_p2p_step)."""
        g = self.rank
        up_rows = self.rows[g - 1][1] - self.rows[g - 1][0] if g > 0 else 0
        self.B.sharp_band_p2p_step(self.sh.ctx, self.windows, g, self.w, self.h, self.row0, self.row1, up_rows, epoch,
                                   params, out, grid_cap)
        return out

    def close(self):
        for p in self._opened:
            self.B.sharp_ipc_close_handle(p)
        self._opened = []
        if self._owned and self.window:
            self.B.sharp_p2p_window_destroy(self.window)
        self.window = 0
