"""CPU model of the TMEM cell bookkeeping of the tm kernels (csrc/ntt_tmr.cuh, csrc/ntt_tms.cuh).

The kernels move the column-phase -> row-phase intermediate of N = R x 4096 (the
4-step split) through per-thread TMEM cells instead of memory.  This test replays their
address formulas and schedules in plain Python and checks, for several rows in a row:
  * every element of the intermediate gets exactly one cell, and the sub-row stage that needs element
    (k, c) reads the cell the column pass that produced (k, c) wrote, from the same TMEM lane;
  * N = 2^16 (one row in TMEM, two alternating layouts): column pass s of row j + 1 writes exactly the
    cells sub-row s of row j has read -- same thread, so no cross-thread ordering is needed for the
    reuse -- and never a cell another sub-row of row j still has to read;
  * N = 2^14 / 2^15 (two row slots): rows j and j + 1 never share a cell.
No GPU: these are the index functions the kernels use, written out independently of them.
"""
import itertools

TT = 256          # threads per team (one sub-row: 256 threads x 16 elements = 4096)


def lane_half(t):
    """team thread t -> (TMEM lane, column half): lane quadrant of its warp, h = t // 128"""
    return t % 128, t // 128


def col16(layout, p, k, h):
    """N = 2^16 (ntt_tmr.cuh): A: 32 k + 16 h + p, B: 32 p + 16 h + k"""
    return 32 * k + 16 * h + p if layout == "A" else 32 * p + 16 * h + k


def test_n65536_cells_cover_the_row_once_per_layout():
    for layout in "AB":
        seen = {}
        for t in range(TT):
            lane, h = lane_half(t)
            for p in range(16):                    # column pass p: column c = 256 p + t
                for k in range(16):
                    cell = (lane, col16(layout, p, k, h))
                    assert cell not in seen, (layout, t, p, k)
                    seen[cell] = (k, 256 * p + t)  # element (k, c) of the row
        assert len(seen) == 65536                 # 128 lanes x 512 columns: the whole TMEM, once
        assert all(0 <= c < 512 for (_, c) in seen)


def test_n65536_stage1_reads_what_the_column_passes_wrote():
    for layout in "AB":
        wrote = {}                                 # cell -> element (k, c) the column passes put there
        for t in range(TT):
            lane, h = lane_half(t)
            for p in range(16):
                for k in range(16):
                    wrote[(lane, col16(layout, p, k, h))] = (k, 256 * p + t)
        for t in range(TT):
            lane, h = lane_half(t)
            for s in range(16):                    # sub-row s, stage 1, thread t: elements 256 a + t
                for a in range(16):
                    assert wrote[(lane, col16(layout, a, s, h))] == (s, 256 * a + t), (layout, t, s, a)


def test_n65536_ping_pong_reuses_exactly_the_consumed_cells():
    # forward: R(j, s) reads {col_j(a, s, h) : a}; C(j+1, s) then writes {col_{j+1}(s, k, h) : k}
    # inverse: C'(j, s) reads {col_j(s, k, h) : k}; R'(j+1, s) then writes {col_{j+1}(a, s, h) : a}
    layouts = ["A", "B", "A", "B", "A"]
    for j in range(len(layouts) - 1):
        cur, nxt = layouts[j], layouts[j + 1]
        for h in (0, 1):
            for s in range(16):
                read_fwd = {col16(cur, a, s, h) for a in range(16)}
                write_fwd = {col16(nxt, s, k, h) for k in range(16)}
                assert read_fwd == write_fwd, (j, s, h)
                read_inv = {col16(cur, s, k, h) for k in range(16)}
                write_inv = {col16(nxt, a, s, h) for a in range(16)}
                assert read_inv == write_inv, (j, s, h)
            # a column pass never overwrites a cell that another sub-row of row j still reads
            for s, s2 in itertools.permutations(range(16), 2):
                assert not ({col16(nxt, s, k, h) for k in range(16)} & {col16(cur, a, s2, h) for a in range(16)})


def test_n65536_one_access_per_row_is_contiguous():
    # layout A: the sub-row read is 16 contiguous columns (one .x16 load), the column-pass write is
    # strided by 32; layout B the other way round
    for h in (0, 1):
        for s in range(16):
            a_read = [col16("A", a, s, h) for a in range(16)]
            assert a_read == list(range(a_read[0], a_read[0] + 16))
            b_write = [col16("B", s, k, h) for k in range(16)]
            assert b_write == list(range(b_write[0], b_write[0] + 16))
            assert [col16("A", s, k, h) for k in range(16)] == [col16("A", s, 0, h) + 32 * k for k in range(16)]
            assert [col16("B", a, s, h) for a in range(16)] == [col16("B", 0, s, h) + 32 * a for a in range(16)]


def col_slot(R, slot, p, k, h):
    """N = R x 4096, R = 4, 8 (ntt_tms.cuh): column 256 h + 16 R slot + R p + k"""
    return 256 * h + 16 * R * slot + R * p + k


def test_small_n_two_slots_never_overlap_and_fit():
    for R in (4, 8):
        cells = {0: set(), 1: set()}
        for slot in (0, 1):
            for t in range(TT):
                lane, h = lane_half(t)
                for p in range(16):
                    for k in range(R):
                        c = col_slot(R, slot, p, k, h)
                        assert 0 <= c < 512
                        assert (lane, c) not in cells[slot]
                        cells[slot].add((lane, c))
        assert not (cells[0] & cells[1])
        # stage 1 of sub-row s reads (a, s) at stride R; a column pass writes R contiguous cells
        for s in range(R):
            assert [col_slot(R, 1, a, s, 0) for a in range(16)] == [col_slot(R, 1, 0, s, 0) + R * a for a in range(16)]
        assert [col_slot(R, 0, 5, k, 1) for k in range(R)] == list(range(col_slot(R, 0, 5, 0, 1), col_slot(R, 0, 5, 0, 1) + R))


def test_team_work_split_covers_every_pass_and_sub_row_once():
    # four teams; team tau: column passes tau + 4 i (i < 4), sub-rows tau + 4 i (i < R / 4)
    for R in (4, 8, 16):
        passes = sorted(tau + 4 * i for tau in range(4) for i in range(4))
        subrows = sorted(tau + 4 * i for tau in range(4) for i in range(R // 4))
        assert passes == list(range(16))
        assert subrows == list(range(R))
