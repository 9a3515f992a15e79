"""Seeded synthetic PairHMM batches shaped like GATK HaplotypeCaller regions.

This module only DRAWS inputs: it holds none of the method's arithmetic
(no transition probabilities, no priors, no likelihoods) and is the one
module both the CUDA path's tests/bench and the oracle tests use
(DESIGN.md "Input recipe"). Everything is addressable by
``(config seed, region id)``, so a rank can generate its own shard and two
runs of the same config produce byte-identical batches.

Workload shape (PAPER.md L22@4659 "the tasks are the pairs of
sequences", L24@575 "PairHMM ... average 189 tasks per batch", one batch per
region):

  per region
    1. a reference segment of iid uniform ACGT with ~5 % of positions inside
       homopolymer runs of 4-10 bases (to exercise indel paths);
    2. H haplotypes: haplotype 0 is the reference, the others carry SNPs at
       ``snp_rate`` and 1-5 bp indels at ``indel_rate``; each is cut to its
       target length N;
    3. R reads, each copied from a random haplotype at a uniform start, with
       per-base substitution errors drawn with the error probability of the
       base's quality bin; ``decoy_frac`` of the reads are random sequence
       (they exercise the FP64 rescue);
    4. base qualities from a binned Illumina-like mix
       {Q37: 85 %, Q23: 9 %, Q12: 4 %, Q6: 2 %}, ``n_rate`` of the read bases
       set to 'N' with Q6;
    5. insertion/deletion qualities 45 (optionally jittered over U{40..45}),
       gap-continuation quality 10;
    6. pairs = all R x H combinations of the region.

The error probabilities of the quality bins below are data-synthesis
constants (the chance the simulated sequencer mis-called a base), written
out as literals; they are not shared with either implementation.
"""
from __future__ import annotations

import dataclasses
from dataclasses import dataclass, field
from typing import Dict, Iterable, List, Optional, Sequence

import numpy as np

BASES = np.frombuffer(b"ACGT", dtype=np.uint8)

# quality bin -> (probability of the bin, probability that the simulated base is wrong)
QUAL_BINS = np.array([37, 23, 12, 6], dtype=np.uint8)
QUAL_BIN_P = np.array([0.85, 0.09, 0.04, 0.02])
QUAL_BIN_ERR = np.array([1.9952623e-4, 5.0118723e-3, 6.3095734e-2, 2.5118864e-1])


@dataclass
class Batch:
    """A batch in the C-ABI layout of include/phmm.h (host numpy arrays)."""

    read_bases: np.ndarray  # uint8, concatenated, 'A','C','G','T','N'
    base_quals: np.ndarray  # uint8 raw Phred, same layout
    ins_quals: np.ndarray
    del_quals: np.ndarray
    gcp_quals: np.ndarray
    read_offsets: np.ndarray  # int64, n_reads + 1
    hap_bases: np.ndarray  # uint8, concatenated
    hap_offsets: np.ndarray  # int64, n_haps + 1
    pairs: np.ndarray  # int32, (n_pairs, 2) = (read_idx, hap_idx)
    meta: Dict = field(default_factory=dict)

    @property
    def n_reads(self) -> int:
        return int(self.read_offsets.size - 1)

    @property
    def n_haps(self) -> int:
        return int(self.hap_offsets.size - 1)

    @property
    def n_pairs(self) -> int:
        return int(self.pairs.shape[0])

    def read_lengths(self) -> np.ndarray:
        return np.diff(self.read_offsets)

    def hap_lengths(self) -> np.ndarray:
        return np.diff(self.hap_offsets)

    def cells(self) -> int:
        """Sum of m*N over pairs -- the paper's cell count (L22@1416)."""
        m = self.read_lengths()[self.pairs[:, 0]]
        n = self.hap_lengths()[self.pairs[:, 1]]
        return int(np.sum(m.astype(np.int64) * n.astype(np.int64)))

    def pair_cells(self) -> np.ndarray:
        m = self.read_lengths()[self.pairs[:, 0]]
        n = self.hap_lengths()[self.pairs[:, 1]]
        return m.astype(np.int64) * n.astype(np.int64)

    def nbytes_inputs(self) -> int:
        return int(sum(a.nbytes for a in (self.read_bases, self.base_quals, self.ins_quals,
                                          self.del_quals, self.gcp_quals, self.read_offsets,
                                          self.hap_bases, self.hap_offsets, self.pairs)))

    def read(self, r: int) -> bytes:
        return bytes(self.read_bases[self.read_offsets[r]:self.read_offsets[r + 1]])

    def hap(self, h: int) -> bytes:
        return bytes(self.hap_bases[self.hap_offsets[h]:self.hap_offsets[h + 1]])

    def subset(self, pair_idx: Sequence[int]) -> "Batch":
        """Same reads/haps, a subset of the pairs (order preserved)."""
        return dataclasses.replace(self, pairs=np.ascontiguousarray(self.pairs[np.asarray(pair_idx)]),
                                   meta=dict(self.meta))


@dataclass
class RegionSpec:
    """Shape of one config; every length field is a (lo, hi) inclusive range."""

    n_haps: tuple = (4, 4)
    n_reads: tuple = (16, 16)
    read_len: tuple = (100, 100)
    hap_len: tuple = (120, 120)  # absolute N range, unless hap_len_factor is set
    hap_len_factor: Optional[tuple] = None  # N ~ U{ceil(f0*m_region) .. floor(f1*m_region)}
    short_read_frac: float = 0.0  # fraction of reads drawn from short_read_len instead
    short_read_len: tuple = (150, 249)
    snp_rate: float = 0.01
    indel_rate: float = 0.001
    decoy_frac: float = 0.0
    n_rate: float = 0.0005
    indel_qual: tuple = (45, 45)
    gcp_qual: int = 10
    fixed_qual: Optional[int] = None  # all base quals = this (long-read stress)
    fixed_err: Optional[float] = None  # substitution rate to use with fixed_qual


# SURVEY.md §8d configs. BASELINE.json "configs" [0..4] = C1..C5.
CONFIGS: Dict[str, Dict] = {
    "C1": dict(n_regions=1, seed=1, spec=RegionSpec(n_haps=(4, 4), n_reads=(16, 16), read_len=(100, 100),
                                                   hap_len=(120, 120)),
               precision="fp64", desc="64 pairs: 100 bp reads x 120 bp haplotypes, FP64"),
    "C2": dict(n_regions=8192, seed=2, spec=RegionSpec(n_haps=(8, 8), n_reads=(16, 16), read_len=(101, 101),
                                                      hap_len=(300, 300), decoy_frac=0.02),
               precision="fp32", desc="1M pairs: 101 bp reads x 300 bp haplotypes, FP32 + FP64 rescue"),
    "C3": dict(n_regions=4096, seed=3, spec=RegionSpec(n_haps=(4, 8), n_reads=(16, 64), read_len=(250, 250),
                                                      hap_len=(250, 500), short_read_frac=0.1,
                                                      short_read_len=(150, 249)),
               precision="fp32", desc="HaplotypeCaller-shaped regions: 250 bp reads x 4-8 haplotypes"),
    "C4": dict(n_regions=256, seed=4, spec=RegionSpec(n_haps=(8, 8), n_reads=(8, 8), read_len=(1000, 1000),
                                                     hap_len=(1500, 1500), snp_rate=0.01, indel_rate=0.0005,
                                                     fixed_qual=20, fixed_err=0.01, n_rate=0.0),
               precision="fp32", desc="long-read stress: 1000 bp reads x 1500 bp haplotypes"),
    "C5": dict(n_regions=262144, seed=5, spec=RegionSpec(n_haps=(8, 8), n_reads=(32, 32), read_len=(100, 250),
                                                        hap_len_factor=(1.0, 2.0)),
               precision="fp32", desc="64M pairs mixed 100-250 bp (sharded across GPUs)"),
}


def _rng(seed: int, region: int) -> np.random.Generator:
    return np.random.Generator(np.random.Philox(np.random.SeedSequence([int(seed), int(region)])))


def _uniform_int(rng, lohi):
    lo, hi = lohi
    return int(rng.integers(lo, hi + 1))


def _reference(rng, length: int) -> np.ndarray:
    ref = BASES[rng.integers(0, 4, size=length)]
    # ~5 % of positions inside homopolymer runs of 4..10
    covered = 0
    target = int(0.05 * length)
    while covered < target and length > 10:
        run = int(rng.integers(4, 11))
        start = int(rng.integers(0, length - run))
        ref[start:start + run] = BASES[int(rng.integers(0, 4))]
        covered += run
    return ref


def _mutate(rng, seq: np.ndarray, snp_rate: float, indel_rate: float) -> np.ndarray:
    out = seq.copy()
    snp = rng.random(out.size) < snp_rate
    if snp.any():
        shift = rng.integers(1, 4, size=int(snp.sum()))
        code = np.searchsorted(BASES, out[snp])
        out[snp] = BASES[(code + shift) % 4]
    n_indel = rng.binomial(out.size, indel_rate) if indel_rate > 0 else 0
    for _ in range(int(n_indel)):
        pos = int(rng.integers(0, out.size))
        ln = int(rng.integers(1, 6))
        if rng.random() < 0.5:  # insertion
            out = np.concatenate([out[:pos], BASES[rng.integers(0, 4, size=ln)], out[pos:]])
        else:
            out = np.concatenate([out[:pos], out[pos + ln:]])
    return out


def gen_region(spec: RegionSpec, seed: int, region: int):
    """One region: (reads, base_q, ins_q, del_q, gcp_q, haps) as lists of uint8 arrays."""
    rng = _rng(seed, region)
    H = _uniform_int(rng, spec.n_haps)
    R = _uniform_int(rng, spec.n_reads)
    m_region = _uniform_int(rng, spec.read_len)
    # haplotype lengths
    if spec.hap_len_factor is not None:
        lo = int(np.ceil(spec.hap_len_factor[0] * m_region))
        hi = int(np.floor(spec.hap_len_factor[1] * m_region))
        n_h = [int(rng.integers(lo, hi + 1)) for _ in range(H)]
    else:
        n_h = [_uniform_int(rng, spec.hap_len) for _ in range(H)]
    ref = _reference(rng, max(n_h) + 64)
    haps = []
    for h in range(H):
        s = ref if h == 0 else _mutate(rng, ref, spec.snp_rate, spec.indel_rate)
        while s.size < n_h[h]:  # deletions may have shortened it
            s = np.concatenate([s, BASES[rng.integers(0, 4, size=n_h[h] - s.size)]])
        haps.append(np.ascontiguousarray(s[:n_h[h]]))
    reads, bq, iq, dq, gq = [], [], [], [], []
    for _ in range(R):
        m = m_region
        if spec.short_read_frac > 0 and rng.random() < spec.short_read_frac:
            m = _uniform_int(rng, spec.short_read_len)
        src = haps[int(rng.integers(0, H))]
        if rng.random() < spec.decoy_frac:
            read = BASES[rng.integers(0, 4, size=m)]
        elif src.size >= m:
            st = int(rng.integers(0, src.size - m + 1))
            read = src[st:st + m].copy()
        else:  # read longer than the haplotype: extend with random sequence
            read = np.concatenate([src, BASES[rng.integers(0, 4, size=m - src.size)]])
        if spec.fixed_qual is not None:
            q = np.full(m, spec.fixed_qual, dtype=np.uint8)
            err = np.full(m, spec.fixed_err if spec.fixed_err is not None else 0.0)
        else:
            b = rng.choice(4, size=m, p=QUAL_BIN_P)
            q = QUAL_BINS[b].copy()
            err = QUAL_BIN_ERR[b]
        wrong = rng.random(m) < err
        if wrong.any():
            code = np.searchsorted(BASES, read[wrong])
            read = read.copy()
            read[wrong] = BASES[(code + rng.integers(1, 4, size=int(wrong.sum()))) % 4]
        if spec.n_rate > 0:
            nn = rng.random(m) < spec.n_rate
            if nn.any():
                read = read.copy()
                read[nn] = ord("N")
                q[nn] = 6
        lo, hi = spec.indel_qual
        if lo == hi:
            iqr = np.full(m, lo, dtype=np.uint8)
            dqr = np.full(m, lo, dtype=np.uint8)
        else:
            iqr = rng.integers(lo, hi + 1, size=m).astype(np.uint8)
            dqr = rng.integers(lo, hi + 1, size=m).astype(np.uint8)
        reads.append(np.ascontiguousarray(read, dtype=np.uint8))
        bq.append(q.astype(np.uint8))
        iq.append(iqr)
        dq.append(dqr)
        gq.append(np.full(m, spec.gcp_qual, dtype=np.uint8))
    return reads, bq, iq, dq, gq, haps


def make_batch(spec: RegionSpec, seed: int, regions: Iterable[int]) -> Batch:
    """Concatenate regions into one batch; pairs are all R x H per region,
    read-major inside a region."""
    R_b, Q_b, I_b, D_b, G_b, H_b = [], [], [], [], [], []
    pairs: List[np.ndarray] = []
    region_of_pair: List[np.ndarray] = []
    nr = nh = 0
    regions = list(regions)
    for reg in regions:
        reads, bq, iq, dq, gq, haps = gen_region(spec, seed, reg)
        R, H = len(reads), len(haps)
        rr, hh = np.meshgrid(np.arange(R, dtype=np.int32) + nr, np.arange(H, dtype=np.int32) + nh, indexing="ij")
        pairs.append(np.stack([rr.ravel(), hh.ravel()], axis=1))
        region_of_pair.append(np.full(R * H, reg, dtype=np.int64))
        R_b += reads; Q_b += bq; I_b += iq; D_b += dq; G_b += gq; H_b += haps
        nr += R
        nh += H
    rl = np.array([r.size for r in R_b], dtype=np.int64)
    hl = np.array([h.size for h in H_b], dtype=np.int64)
    ro = np.zeros(rl.size + 1, dtype=np.int64); np.cumsum(rl, out=ro[1:])
    ho = np.zeros(hl.size + 1, dtype=np.int64); np.cumsum(hl, out=ho[1:])
    cat = lambda xs: np.ascontiguousarray(np.concatenate(xs) if xs else np.zeros(0, np.uint8), dtype=np.uint8)
    return Batch(read_bases=cat(R_b), base_quals=cat(Q_b), ins_quals=cat(I_b), del_quals=cat(D_b),
                 gcp_quals=cat(G_b), read_offsets=ro, hap_bases=cat(H_b), hap_offsets=ho,
                 pairs=np.ascontiguousarray(np.concatenate(pairs) if pairs else np.zeros((0, 2), np.int32),
                                            dtype=np.int32),
                 meta=dict(seed=seed, regions=(regions[0], regions[-1] + 1) if regions else (0, 0),
                           region_of_pair=np.concatenate(region_of_pair) if region_of_pair else None))


def config_batch(name: str, n_regions: Optional[int] = None, region_start: int = 0, seed: Optional[int] = None,
                 **spec_overrides) -> Batch:
    """The batch of config ``name`` (C1..C5), optionally only ``n_regions``
    regions starting at ``region_start`` (a shard, or a reduced test size)."""
    c = CONFIGS[name]
    spec = dataclasses.replace(c["spec"], **spec_overrides) if spec_overrides else c["spec"]
    nreg = c["n_regions"] if n_regions is None else n_regions
    b = make_batch(spec, c["seed"] if seed is None else seed, range(region_start, region_start + nreg))
    b.meta["config"] = name
    return b


def random_pairs_batch(seed: int, n_pairs: int, m_range=(1, 40), n_range=(1, 60), qual_range=(0, 60),
                       indel_qual_range=(10, 60), gcp_range=(5, 40), n_frac=0.05) -> Batch:
    """Unstructured random pairs (every read its own haplotype): edge-case
    coverage for parity tests -- ragged lengths, Q0, N bases, m > N."""
    rng = _rng(seed, 0)
    alphabet = np.frombuffer(b"ACGTN", dtype=np.uint8)
    p = np.array([(1 - n_frac) / 4] * 4 + [n_frac])
    reads, bq, iq, dq, gq, haps = [], [], [], [], [], []
    for _ in range(n_pairs):
        m = int(rng.integers(m_range[0], m_range[1] + 1))
        n = int(rng.integers(n_range[0], n_range[1] + 1))
        reads.append(alphabet[rng.choice(5, size=m, p=p)])
        haps.append(alphabet[rng.choice(5, size=n, p=p)])
        bq.append(rng.integers(qual_range[0], qual_range[1] + 1, size=m).astype(np.uint8))
        iq.append(rng.integers(indel_qual_range[0], indel_qual_range[1] + 1, size=m).astype(np.uint8))
        dq.append(rng.integers(indel_qual_range[0], indel_qual_range[1] + 1, size=m).astype(np.uint8))
        gq.append(rng.integers(gcp_range[0], gcp_range[1] + 1, size=m).astype(np.uint8))
    rl = np.array([r.size for r in reads], dtype=np.int64)
    hl = np.array([h.size for h in haps], dtype=np.int64)
    ro = np.zeros(n_pairs + 1, dtype=np.int64); np.cumsum(rl, out=ro[1:])
    ho = np.zeros(n_pairs + 1, dtype=np.int64); np.cumsum(hl, out=ho[1:])
    cat = lambda xs: np.ascontiguousarray(np.concatenate(xs) if xs else np.zeros(0, np.uint8), dtype=np.uint8)
    idx = np.arange(n_pairs, dtype=np.int32)
    return Batch(read_bases=cat(reads), base_quals=cat(bq), ins_quals=cat(iq), del_quals=cat(dq),
                 gcp_quals=cat(gq), read_offsets=ro, hap_bases=cat(haps), hap_offsets=ho,
                 pairs=np.ascontiguousarray(np.stack([idx, idx], axis=1)), meta=dict(seed=seed))


def concat_batches(batches: Sequence[Batch]) -> Batch:
    """Concatenate batches (indices re-based)."""
    ro_parts, ho_parts, pairs = [np.zeros(1, np.int64)], [np.zeros(1, np.int64)], []
    r_base = h_base = 0
    rb_off = hb_off = 0
    for b in batches:
        ro_parts.append(b.read_offsets[1:] + rb_off)
        ho_parts.append(b.hap_offsets[1:] + hb_off)
        pairs.append(b.pairs + np.array([r_base, h_base], dtype=np.int32))
        r_base += b.n_reads
        h_base += b.n_haps
        rb_off += int(b.read_offsets[-1])
        hb_off += int(b.hap_offsets[-1])
    cat = lambda name: np.ascontiguousarray(np.concatenate([getattr(b, name) for b in batches]), dtype=np.uint8)
    return Batch(read_bases=cat("read_bases"), base_quals=cat("base_quals"), ins_quals=cat("ins_quals"),
                 del_quals=cat("del_quals"), gcp_quals=cat("gcp_quals"),
                 read_offsets=np.concatenate(ro_parts), hap_bases=cat("hap_bases"),
                 hap_offsets=np.concatenate(ho_parts),
                 pairs=np.ascontiguousarray(np.concatenate(pairs), dtype=np.int32))


# ---------------------------------------------------------------- Smith-Waterman tasks
@dataclass
class SwBatch:
    """Smith-Waterman tasks in the C-ABI layout of include/phmm.h (phmm_sw_batch)."""

    ref_bases: np.ndarray   # uint8 rows sequences, concatenated
    ref_offsets: np.ndarray  # int64, n_refs + 1
    alt_bases: np.ndarray   # uint8 column sequences
    alt_offsets: np.ndarray  # int64, n_alts + 1
    tasks: np.ndarray       # int32 (n_tasks, 2): (ref_idx, alt_idx)
    meta: dict = field(default_factory=dict)

    @property
    def n_tasks(self) -> int:
        return int(self.tasks.shape[0])

    def ref(self, r: int) -> bytes:
        return self.ref_bases[self.ref_offsets[r]:self.ref_offsets[r + 1]].tobytes()

    def alt(self, a: int) -> bytes:
        return self.alt_bases[self.alt_offsets[a]:self.alt_offsets[a + 1]].tobytes()

    def cells(self) -> int:
        t = self.tasks
        m = self.ref_offsets[t[:, 0] + 1] - self.ref_offsets[t[:, 0]]
        n = self.alt_offsets[t[:, 1] + 1] - self.alt_offsets[t[:, 1]]
        return int(np.sum(m.astype(np.int64) * n))

    def ops_capacity(self) -> np.ndarray:
        """Per-task CIGAR capacity offsets (prefix sums of M + N), the ABI's layout."""
        t = self.tasks
        cap = (self.ref_offsets[t[:, 0] + 1] - self.ref_offsets[t[:, 0]]) + \
              (self.alt_offsets[t[:, 1] + 1] - self.alt_offsets[t[:, 1]])
        return np.concatenate([[0], np.cumsum(cap)]).astype(np.int64)


# The paper's SW workload: per HaplotypeCaller region, each candidate haplotype is aligned
# against the reference window (L16@3860: "the algorithm has been modified to adapt to the
# needs of HaplotypeCaller"); batches average four tasks (L24@560) and were re-batched to
# 3,200 tasks (L24@1700). SW1 = that re-batched size, SW2 = a large batch.
SW_CONFIGS = {
    "SW1": dict(n_regions=800, n_haps=4, window=(300, 500), seed=21,
                desc="3,200 tasks: 4 haplotypes x 800 regions against 300-500 bp reference windows"),
    "SW2": dict(n_regions=16384, n_haps=4, window=(300, 500), seed=22,
                desc="65,536 tasks: 4 haplotypes x 16,384 regions, 300-500 bp windows"),
}


def sw_region(seed: int, region: int, n_haps: int, window) -> tuple:
    """One region: the reference window and n_haps haplotypes (SNPs 1 %, 1-5 bp indels
    0.5 %, so the alignments have gaps)."""
    rng = _rng(seed, region)
    w = _uniform_int(rng, window)
    ref = _reference(rng, w)
    haps = [_mutate(rng, ref, 0.01, 0.005) for _ in range(n_haps)]
    return ref, haps


def sw_config_batch(name: str, n_regions: Optional[int] = None, seed: Optional[int] = None) -> SwBatch:
    cfg = SW_CONFIGS[name]
    R = cfg["n_regions"] if n_regions is None else n_regions
    s = cfg["seed"] if seed is None else seed
    refs, alts, tasks = [], [], []
    for reg in range(R):
        ref, haps = sw_region(s, reg, cfg["n_haps"], cfg["window"])
        refs.append(ref)
        for h in haps:
            tasks.append((len(refs) - 1, len(alts)))
            alts.append(h)
    return _sw_pack(refs, alts, tasks, dict(config=name, seed=s, n_regions=R))


def sw_random_batch(seed: int, n_tasks: int, m_range=(1, 60), n_range=(1, 60), alphabet=b"ACGTN",
                    related: float = 0.5) -> SwBatch:
    """Ragged random tasks for parity edge cases; a fraction `related` of the columns
    sequences are mutated copies of their row sequence (long alignments with gaps)."""
    rng = _rng(seed, 0)
    alph = np.frombuffer(alphabet, dtype=np.uint8)
    refs, alts, tasks = [], [], []
    for t in range(n_tasks):
        m = int(rng.integers(m_range[0], m_range[1] + 1))
        n = int(rng.integers(n_range[0], n_range[1] + 1))
        a = alph[rng.integers(0, alph.size, size=m)]
        if rng.random() < related:
            b = _mutate(rng, np.where(a == ord("N"), ord("A"), a).astype(np.uint8), 0.05, 0.03)[:n]
            if b.size < n:
                b = np.concatenate([b, alph[rng.integers(0, alph.size, size=n - b.size)]])
        else:
            b = alph[rng.integers(0, alph.size, size=n)]
        refs.append(a.astype(np.uint8))
        alts.append(b.astype(np.uint8))
        tasks.append((t, t))
    return _sw_pack(refs, alts, tasks, dict(seed=seed))


def _sw_pack(refs, alts, tasks, meta) -> SwBatch:
    ro = np.zeros(len(refs) + 1, dtype=np.int64)
    np.cumsum([r.size for r in refs], out=ro[1:])
    ao = np.zeros(len(alts) + 1, dtype=np.int64)
    np.cumsum([a.size for a in alts], out=ao[1:])
    cat = lambda xs: np.ascontiguousarray(np.concatenate(xs) if xs else np.zeros(0, np.uint8), dtype=np.uint8)
    return SwBatch(ref_bases=cat(refs), ref_offsets=ro, alt_bases=cat(alts), alt_offsets=ao,
                   tasks=np.ascontiguousarray(np.asarray(tasks, dtype=np.int32).reshape(-1, 2)), meta=meta)
