"""Multi-GPU sharding of the batched RNS NTT (SURVEY.md 8 row e).

RNS limbs and polynomials are independent transforms (the RNS
dimension L is a parallel axis of every ciphertext), so the path shards with
NO collective inside the transform.  Two partitionings:

* limb shard  (config 4): rank g owns limbs [l0, l1) = limb_range(L, G, g) and
  builds its own plan with that prime subset (its twiddle tables shrink by G);
* batch shard (config 3 weak scaling): rank g owns its own polynomials.

NCCL (``torch.distributed``, backend "nccl" on GPUs, "gloo" in the CPU tests)
is used only to scatter inputs before and gather results after, for workloads
that start or end on one rank.  The transform itself is a callable so the
host logic can be exercised on CPU; on the GPU it is ``wdntt.Plan.forward``.
"""
from __future__ import annotations

from typing import Callable

import torch
import torch.distributed as dist


def limb_range(L: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous, balanced limb range of ``rank`` (sizes differ by at most 1)."""
    base, extra = divmod(L, world)
    l0 = rank * base + min(rank, extra)
    return l0, l0 + base + (1 if rank < extra else 0)


def scatter_limbs(x_full: torch.Tensor | None, L: int, N: int, batch: int, src: int = 0) -> torch.Tensor:
    """Rank ``src`` holds [batch][L][N]; every rank receives its [batch][L_g][N] limb slice.

    The limb slices of a [B][L][N] array are strided, so rank ``src`` first makes
    each slice contiguous (one copy), then ``dist.scatter`` moves them.
    """
    world, rank = dist.get_world_size(), dist.get_rank()
    l0, l1 = limb_range(L, world, rank)
    dev = x_full.device if x_full is not None else None
    sizes = [limb_range(L, world, g) for g in range(world)]
    maxl = max(b - a for a, b in sizes)
    # scatter needs equal-size chunks: pad each slice to maxl limbs
    recv = torch.empty((batch, maxl, N), dtype=torch.int32, device=dev if dev is not None else _device())
    if rank == src:
        chunks = []
        for a, b in sizes:
            c = torch.zeros((batch, maxl, N), dtype=torch.int32, device=x_full.device)
            c[:, : b - a] = x_full[:, a:b]
            chunks.append(c)
        dist.scatter(recv, chunks, src=src)
    else:
        dist.scatter(recv, None, src=src)
    return recv[:, : l1 - l0].contiguous()


def gather_limbs(y_local: torch.Tensor, L: int, N: int, batch: int, dst: int = 0) -> torch.Tensor | None:
    """Inverse of ``scatter_limbs``: rank ``dst`` gets the full [batch][L][N]."""
    world, rank = dist.get_world_size(), dist.get_rank()
    sizes = [limb_range(L, world, g) for g in range(world)]
    maxl = max(b - a for a, b in sizes)
    send = torch.zeros((batch, maxl, N), dtype=torch.int32, device=y_local.device)
    send[:, : y_local.shape[1]] = y_local
    if rank == dst:
        bufs = [torch.empty_like(send) for _ in range(world)]
        dist.gather(send, bufs, dst=dst)
        out = torch.empty((batch, L, N), dtype=torch.int32, device=y_local.device)
        for (a, b), buf in zip(sizes, bufs):
            out[:, a:b] = buf[:, : b - a]
        return out
    dist.gather(send, None, dst=dst)
    return None


def sharded_transform(x_full: torch.Tensor | None, primes: list[int], N: int, batch: int,
                      transform: Callable[[torch.Tensor, list[int]], torch.Tensor],
                      src: int = 0) -> torch.Tensor | None:
    """scatter limbs -> local transform on this rank's primes -> gather to ``src``."""
    world, rank = dist.get_world_size(), dist.get_rank()
    l0, l1 = limb_range(len(primes), world, rank)
    xl = scatter_limbs(x_full, len(primes), N, batch, src)
    yl = transform(xl, primes[l0:l1]) if l1 > l0 else xl
    return gather_limbs(yl, len(primes), N, batch, src)


def _device():
    return torch.device("cuda", torch.cuda.current_device()) if torch.cuda.is_available() and \
        dist.get_backend() == "nccl" else torch.device("cpu")


def sharded_modup(x_local: torch.Tensor, partial_fn: Callable[[torch.Tensor], torch.Tensor],
                  finish_fn: Callable[[torch.Tensor], torch.Tensor]) -> torch.Tensor:
    """Limb-sharded ModUp (SURVEY.md 8 rows e + f3): the one exchange step of the path.

    Every rank holds its shard of the Q limbs ``x_local`` [B][a_g][N] (NTT domain).
    ``partial_fn`` returns this shard's share of BConv_{Q->P} as int64 [B][k][N]
    (on the GPU: ``RnsConv.modup_partial`` of a shard conversion object); the shares are
    summed by ONE all-reduce, then ``finish_fn`` reduces mod p_j and NTTs
    (``RnsConv.modup_finish``).  Returns the P limbs [B][k][N], identical on every rank.
    The all-reduce moves B*k*N*8 bytes per rank: k = 1 special prime (Table III)
    makes it 1/a of the input.
    """
    part = partial_fn(x_local)
    dist.all_reduce(part, op=dist.ReduceOp.SUM)
    return finish_fn(part)
