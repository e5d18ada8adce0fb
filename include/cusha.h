/*
 * cusha.h — C ABI of the B200-native CuSha shard-processing path.
 *
 * Paper: F. Khorasani, K. Vora, R. Gupta, L. N. Bhuyan, "CuSha: Vertex-Centric
 * Graph Processing on GPUs", HPDC'14.  Citations "L<n>" are lines of the
 * paper text with the section / figure / table they fall in.
 *
 * Problem statement (L45, §4): the user picks a
 * vertex-centric algorithm (Table 3: a Vertex / StaticVertex / Edge
 * type and init_compute / compute / update_condition); CuSha lays the graph
 * out as G-Shards (§3.1) or Concatenated Windows (§3.2),
 * chooses the shard size itself (L310), iterates the 4-stage shard pass
 * (Fig. 5) until an iteration commits no update (L189), and returns
 * the final vertex values (copied to the host only at the end, L457).  The
 * eight Table-3 algorithms are compiled in; the ABI selects one by enum.
 *
 * Conventions for every entry point:
 *  - Plain C types only.  Pointers documented "host" are ordinary host
 *    memory; "device" pointers are CUDA device pointers on opts->device.
 *  - Return value: CUSHA_OK (0) or a positive informational code on success,
 *    a negative CUSHA_E* code on failure; cusha_last_error() then returns a
 *    thread-local message.  No exception or longjmp crosses the ABI.
 *  - The library never reads caller memory after a call returns.
 *  - Thread safety: distinct graphs may be used from distinct threads; one
 *    graph must not be used concurrently.
 *  - Limits: |V| < 2^31, |E| < 2^32 - 2^26 (offsets are 32-bit), and
 *    vertices_per_shard <= 65534 (16-bit local indices).
 *  - Fixed-point range (PR, NN, HS, CS): stage 2 sums the per-edge terms of
 *    Table 3 as 64-bit fixed point with 32 fraction bits (order-independent,
 *    DESIGN.md R11).  Each term is truncated toward zero to a multiple of
 *    2^-32 (so a vertex's sum is within in-degree * 2^-32 of the exact sum of
 *    its f32 terms) and every sum must stay below 2^31 in magnitude.  PR meets
 *    this by construction (the ranks sum to at most |V| < 2^31 at every pass);
 *    for NN / HS / CS cusha_run returns CUSHA_EINVAL when max|initial value| x
 *    max|edge value| x max in-degree (NN: max(|x0|, 1) * |w|; HS: 2 |Q0| |c|;
 *    CS: max(|V0|, 1) * max(|G|, 1)) reaches 2^31 or is not finite.
 */
#ifndef CUSHA_H
#define CUSHA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#if defined(__GNUC__)
#define CUSHA_API __attribute__((visibility("default")))
#else
#define CUSHA_API
#endif

#define CUSHA_ABI_VERSION 5

/* Return codes. */
enum {
  CUSHA_OK = 0,
  CUSHA_NOT_CONVERGED = 1,   /* max_iters reached; values of the last iteration are retrievable */
  CUSHA_EINVAL = -1,         /* bad argument (null pointer, id out of range, size mismatch, ...) */
  CUSHA_ENOMEM = -2,         /* device or host allocation failed */
  CUSHA_ECUDA = -3,          /* CUDA runtime error (message names the call) */
  CUSHA_ENCCL = -4,          /* NCCL error (multi-GPU) */
  CUSHA_EUNSUPPORTED = -5,   /* feature not available in this build / configuration */
  CUSHA_ESTATE = -6          /* call out of order (e.g. get_values before any run) */
};

/* The eight benchmark algorithms of Table 3 (L314-325), in the table's order. */
typedef enum {
  CUSHA_BFS = 0,   /* Vertex {u32 Level};           L316 */
  CUSHA_SSSP = 1,  /* Vertex {u32 Dist}, Edge {u32 Weight}; L317, Fig. 6 */
  CUSHA_PR = 2,    /* Vertex {f32 Rank}, StaticVertex {u32 NbrsNum}; L318 */
  CUSHA_CC = 3,    /* Vertex {u32 Cmpnent};         L319 */
  CUSHA_SSWP = 4,  /* Vertex {u32 BWidth}, Edge {u32 Width}; L320 */
  CUSHA_NN = 5,    /* Vertex {f32 x}, Edge {f32 Weight}; L321 */
  CUSHA_HS = 6,    /* Vertex {f32 Q, f32 Q_new}, Edge {f32 coeff}; L322 */
  CUSHA_CS = 7     /* Vertex {f32 V, f32 GsumOrA}, Edge {f32 G}; L323 */
} cusha_algorithm;

/* Graph representation (§3.1 G-Shards, §3.2 Concatenated Windows). */
typedef enum { CUSHA_REPR_GSHARDS = 0, CUSHA_REPR_CW = 1 } cusha_repr;

/* Where cusha_build_graph's src/dst/edge_values live. */
typedef enum { CUSHA_INPUT_HOST = 0, CUSHA_INPUT_DEVICE = 1 } cusha_input_location;

typedef struct {
  cusha_repr repr;                 /* G-Shards or CW (default G-Shards)                        */
  uint32_t vertices_per_shard;     /* |N|; 0 = the paper's rule (L310, cusha_shard_size)       */
  uint32_t smem_bytes_per_vertex;  /* sizeof(Vertex) assumed by the |N| rule; 0 = 4 (L310)     */
  int device;                      /* CUDA device ordinal                                      */
  void* stream;                    /* cudaStream_t to run on; NULL = a library-owned stream    */
  cusha_input_location input_location; /* host (copied in, timed as H2D) or device            */
  int host_loop;                   /* 0 = loop on the device (default);
                                      1 = host launches passes in chunks of 16 (one launch per
                                      pass, for profilers); passes past convergence exit at once,
                                      so results are identical                                */
  /* Destination-range partition (row e; north_star (4)).  With
   * world_size = G > 1 the shards are split into G contiguous ranges of
   * near-equal work (cusha_partition_shards); partition r owns the vertices
   * of its shards.  Within a partition the pass is asynchronous (L45); across
   * partitions it is BSP: every pass of every partition ends before the next
   * pass starts anywhere.  Each partition keeps only its own shards (the
   * in-edges of its vertices) and the Concatenated Windows of its own source
   * shards; stage 4 of a source shard stores each window's new SrcValues
   * directly into the SrcValue array of the partition that owns the window
   * (the windows aimed at one partition are one contiguous segment of CW_i,
   * L175).  Only shards that committed an update write back (Fig. 5 line 23),
   * and the integer algorithms store only changed vertices, so the exchange is
   * exactly the changed values, overlapped with the other shards' work.
   * After each pass the partitions' "committed an update" words are OR-ed:
   * the global convergence test of L189.  CW representation only.
   *   One process per GPU (nccl_unique_id != NULL, or transport IPC): every
   *     rank passes the full edge list and its rank; it builds only its own
   *     partition.  The ranks map each other's SrcValue, dirty[], barrier
   *     block and VertexValues with CUDA IPC (see `transport`), so stage-4
   *     stores travel over NVLink / NVSwitch and the per-pass OR and barrier
   *     are stores and system-scope atomics in peer memory.  Every rank must
   *     make the same sequence of calls (build, run, get_values).
   *   nccl_unique_id == NULL (transport NCCL): all G partitions run in this process on one
   *     device (each partition with its own arrays, the same kernels and the
   *     same stores into the sibling partitions' SrcValue; the OR is a kernel
   *     over the partitions' words).  Used to test the partitioned algorithm
   *     on one GPU.                                                            */
  int world_size;                  /* 1 = single partition (0 is treated as 1)                  */
  int rank;                        /* this process's rank, 0..world_size-1 (one process per GPU) */
  const void* nccl_unique_id;      /* 128-byte ncclUniqueId, or NULL (see above)                */
  /* Clean-shard skipping (opt-in; not in the paper, which processes every
   * shard in every iteration, Fig. 5 line 3 / L189).  1: a shard none of whose
   * windows was written since its own last pass is skipped — it would
   * recompute the values it holds and commit nothing (exact for all eight
   * algorithms; HS shards that committed re-run, their local state reads
   * their own Q).  Results are identical; passes can differ only in that
   * skipped shards do no work.  cusha_stats.edges_processed counts the edges
   * actually streamed.  Default 0 = the paper's full passes.              */
  int skip_clean_shards;
  /* Host-streamed topology (row f3; the multi-streamed procedure of L455 for
   * graphs whose representation does not fit in HBM).  0 = every array in HBM
   * (default).  Otherwise at most this many bytes of HBM hold the per-entry
   * topology arrays (DestIndex, EdgeValue, SrcIndex, edge ids; CW: SrcIndexCW,
   * Mapper): shards 0..h-1 keep theirs in HBM, shards h..S-1 (h =
   * cusha_stats.host_shard) keep theirs in pinned, mapped host memory, and
   * every pass streams them over the host link through the same TMA ring that
   * streams HBM tiles, overlapping the transfer with the shard computation.
   * SrcValue, VertexValues and the O(|V| + |S|^2) arrays stay in HBM.  Results
   * are identical to the in-HBM layout.  The build itself runs in HBM first.  */
  uint64_t device_topology_budget;
  /* Iteration boundary of the device loop (row a5; DESIGN.md "Overlapped
   * passes").
   *  2 = overlapped passes: one launch runs every pass; shards are drawn as
   *      tickets across passes, so a CTA done with its part of pass k starts
   *      pass k+1 (the asynchronous model of L45 carried across the iteration
   *      boundary; a shard's passes stay in order).  Convergence is concluded
   *      only from a pass that started after every earlier pass completed and
   *      committed nothing (L189), so results are those of the barrier mode.
   *  1 = one launch per pass under a CUDA-graph while node, with a
   *      device-wide barrier between passes as in Fig. 5.
   *  0 (default) = automatic: 2, except with many small shards (>= 16 shards
   *      per resident CTA and <= 16384 entries per shard on average), where
   *      the per-ticket costs of overlapped passes outweigh the barrier they
   *      save and the run uses 1 (measured).
   * host_loop = 1 or world_size > 1 imply one launch per pass.  Other values:
   * CUSHA_EINVAL.  One launch per pass is a fixed-count CUDA graph of 16
   * passes per host check (passes past convergence exit at once).        */
  int pass_barrier;
  /* 1 = keep arrays that only layout inspection (cusha_get_layout) reads:
   * the input edge index of every shard entry and, for CW, the window
   * table.  0 (default) = release them after the build.                    */
  int keep_layout;
  /* Schedule of SrcValue visibility (SURVEY.md §8(b) cusha_mode; L45, L433).
   * CUSHA_MODE_ASYNC (0, default, the paper's): a shard's stage-4 write-back
   *   is visible to shards processed after it in the same pass.
   * CUSHA_MODE_BSP (1, two-phase): every pass reads the SrcValues as they were
   *   at the end of the previous pass (stage 4 writes a second copy that the
   *   next pass reads); the pass sequence is then deterministic and matches
   *   the oracle's mode T pass for pass (tests/test_gpu_bsp.py).  Single
   *   partition only; one launch per pass plus a copy of SrcValue.         */
  int mode;
  /* One process per GPU: how long (ms) a rank waits for its peers (the NCCL
   * bootstrap, a pass barrier) before it gives up and returns CUSHA_ENCCL
   * (an NCCL asynchronous error aborts the bootstrap at once).  0 = 300000.  */
  uint32_t comm_timeout_ms;
  /* One process per GPU: how the ranks find each other's arrays.
   * CUSHA_TRANSPORT_NCCL (0): with nccl_unique_id, cusha_build_graph
   *   all-gathers the ranks' CUDA IPC handles over NCCL.
   * CUSHA_TRANSPORT_IPC (1): no NCCL at all; after cusha_build_graph every
   *   rank passes cusha_ipc_export's blob to the others (e.g. an all-gather
   *   over torch.distributed) and calls cusha_ipc_connect with all of them.
   * In both, everything after the bootstrap is peer memory: stage-4 stores
   * into the owning rank's SrcValue, a per-pass barrier and convergence vote
   * through the ranks' barrier blocks, and cusha_get_values reading every
   * rank's slice.  Ranks may share one device (then the stores stay in HBM).  */
  int transport;
} cusha_build_opts;

enum { CUSHA_TRANSPORT_NCCL = 0, CUSHA_TRANSPORT_IPC = 1 };
#define CUSHA_IPC_BLOB_BYTES 256  /* cusha_ipc_export: four 64-byte cudaIpcMemHandle_t */

enum { CUSHA_MODE_ASYNC = 0, CUSHA_MODE_BSP = 1 };

typedef struct cusha_graph cusha_graph;   /* opaque; owns all device memory it allocates */

typedef struct {
  uint32_t num_vertices;
  uint64_t num_edges;
  uint32_t vertices_per_shard;     /* |N| actually used                                        */
  uint32_t num_shards;             /* |S| = ceil(|V| / |N|) (L173)                             */
  uint32_t repr;                   /* cusha_repr                                               */
  int32_t last_algorithm;          /* -1 before the first run                                  */
  uint32_t iterations;             /* shard passes of the last run (incl. the converged one)   */
  uint32_t converged;              /* 1 if the last run's final pass committed nothing         */
  double build_ms;                 /* cusha_build_graph wall time on the stream (incl. H2D)    */
  double h2d_ms;                   /* build start to the last host-input copy landing (the copies
                                      overlap the first layout pass, row f2)                   */
  double run_ms;                   /* last cusha_run: init + all shard passes (device events)  */
  double loop_ms;                  /* last cusha_run: the shard passes only (device events)    */
  uint64_t h2d_bytes;              /* bytes copied host->device by the build                   */
  uint64_t device_bytes;           /* topology + value arrays resident on the device           */
  uint64_t entries_padded;         /* shard entries incl. vector padding                       */
  uint64_t stage2_bytes_per_iter;  /* algorithmic bytes stage 2 streams per iteration          */
  uint64_t wb_bytes_all_active;    /* stage-4 algorithmic bytes if every shard is active       */
  uint64_t algorithmic_bytes;      /* last run: sum over iterations of stage1..4 algorithmic bytes */
  uint64_t edges_processed;        /* last run: edges streamed by stage 2 over all passes of this
                                      process's shards (iterations * |E| unless shards were
                                      skipped or partitioned)                                 */
  uint32_t device_loop;            /* 0 = passes launched by the host; 1 = CUDA-graph while node,
                                      one launch per pass; 2 = overlapped passes, one launch    */
  int world_size, rank;
  uint64_t host_bytes;             /* per-entry topology bytes held in pinned host memory (f3)  */
  uint32_t host_shard;             /* first shard whose topology is host-resident (|S|: none)   */
  uint32_t mapper_form;            /* last run, CW: 1 = stage 4 used the Mapper in window form
                                      (u16 window index per entry + per-shard delta row), 0 = u32 Mapper */
  uint64_t paper_bytes;            /* last run: algorithmic bytes in the paper's layout (4-byte
                                      fields: stage 2 8/12/16 B per edge, stage 4
                                      CW 12 / GS 8 B (+4 for 8-byte Vertex) per active edge,
                                      2 x sizeof(Vertex) per vertex)                            */
  uint64_t wb_entries;             /* last run: stage-4 entries visited (active shards' windows) */
  uint64_t vertices_processed;     /* last run: vertices of the processed shards, over all passes */
  uint64_t updated_total;          /* last run: committed updates, over all passes               */
  uint32_t partitions;             /* partitions of the graph (row e); 1 = unpartitioned         */
  uint32_t max_in_degree;          /* largest in-degree (fixed-point range check)                */
  uint64_t max_part_device_bytes;  /* the largest partition's device_bytes (= device_bytes at 1)  */
  uint32_t ring_slots;             /* last run: TMA ring slots per CTA of the shard pass          */
  uint32_t l2_read_ahead;          /* last run: 1 = stage-2 tiles were prefetched into L2 ahead of
                                      the ring (a pass streams more than twice the L2)          */
} cusha_stats;

/* ---------------------------------------------------------------- build */
/*
 * Build the G-Shards / CW representation of a directed graph (row a0).
 *   num_vertices, num_edges  |V|, |E|.
 *   src, dst                 edge endpoints, num_edges each, values < num_vertices
 *                            (host or device per opts->input_location; caller-owned,
 *                            read only during the call).  An edge u->v is stored in
 *                            the shard that owns v (incoming edges, L119).
 *   edge_values              nullable; num_edges raw 4-byte values: u32 Weight (SSSP),
 *                            u32 Width (SSWP) or f32 bits (NN Weight, HS coeff, CS G).
 *   opts                     nullable = defaults.
 *   out                      receives the graph handle.
 * Layout (L119-179): shard s owns vertices [s*|N|, (s+1)*|N|); its entries are
 * sorted by (SrcIndex, DestIndex, input order) (Ordered L129; tie-break DESIGN.md
 * R17); window W_ij (L155) and, for CW, CW_i and Mapper (L175) are derived from
 * that order.  |N| = opts->vertices_per_shard or the L310 rule.  Duplicates and
 * self-loops are kept as separate edges (R22).
 * Errors: CUSHA_EINVAL (null src/dst/out with |E|>0, |V|=0, endpoint >= |V|,
 * limits), CUSHA_ENOMEM, CUSHA_ECUDA.
 */
CUSHA_API int cusha_build_graph(uint32_t num_vertices, uint64_t num_edges, const uint32_t* src, const uint32_t* dst,
                      const uint32_t* edge_values, const cusha_build_opts* opts, cusha_graph** out);

/* Release every resource of g (NULL is ignored). */
CUSHA_API void cusha_free_graph(cusha_graph* g);

/*
 * Initial vertex values for the next cusha_run of `alg` (host pointer, copied).
 * Required for NN (f32 x0[|V|]), HS (f32 Q0[|V|]) and CS (f32 pairs
 * {V0, GsumOrA0}[|V|]; GsumOrA0 != 0 marks an anchor, R15).  Optional for the
 * others (overrides the Table-3 start state; e.g. to resume).  bytes must equal
 * |V| * cusha_value_bytes(alg).  Errors: CUSHA_EINVAL.
 */
CUSHA_API int cusha_set_vertex_values(cusha_graph* g, cusha_algorithm alg, const void* init, size_t bytes);

/* ------------------------------------------------------------------ run */
/*
 * Run `alg` to convergence (rows a1-a5): initialise VertexValues (Table 3
 * start state, L327) and every SrcValue copy (R20), then repeat the shard
 * pass (Fig. 5) until a pass commits no update (L189) or max_iters passes ran.
 *   source     BFS/SSSP/SSWP start vertex (< |V|); ignored by the others.
 *   max_iters  upper bound on shard passes (R23); 0 = do nothing.
 * The iteration loop runs on the device (one launch of overlapped passes by
 * default); the host waits once at the end.
 * Returns CUSHA_OK, CUSHA_NOT_CONVERGED, or CUSHA_EINVAL (bad source, NN/HS/CS
 * without initial values, EdgeValue needed but absent) / CUSHA_ECUDA.
 */
CUSHA_API int cusha_run(cusha_algorithm alg, cusha_graph* g, uint32_t source, uint32_t max_iters);

/*
 * Copy the last run's VertexValues (|V| * cusha_value_bytes(alg) bytes) to
 * `out` (host) / `dptr` (device).  Element types: u32 Level / Dist / Cmpnent /
 * BWidth (INF = 0xFFFFFFFF, R1); f32 Rank / x; {f32 Q, f32 Q_new};
 * {f32 V, f32 GsumOrA}.  out_bytes must be exactly that size.
 * Errors: CUSHA_EINVAL (size), CUSHA_ESTATE (no run yet).
 */
CUSHA_API int cusha_get_values(const cusha_graph* g, void* out, size_t out_bytes);
CUSHA_API int cusha_get_values_device(const cusha_graph* g, void* dptr, size_t out_bytes);

/* Statistics of the graph and of its last run (host struct, filled). */
CUSHA_API int cusha_get_stats(const cusha_graph* g, cusha_stats* s);

/*
 * Per-iteration trace of the last run (row f4 / Fig. 7): for i <
 * min(iterations, cap): updated_vertices[i] (committed updates) and
 * active_shards[i] (shards that ran stage 4).  Either pointer may be NULL.
 * Returns the number of iterations written.
 */
CUSHA_API int cusha_get_trace(const cusha_graph* g, uint32_t* updated_vertices, uint32_t* active_shards, uint32_t cap);

/* ------------------------------------------------------- layout export */
/* Device arrays of the representation, copied to host for inspection/tests.
 * Positions are "padded": each shard's (and each CW_i's) entries start at a
 * multiple of 8 and are followed by filler entries up to the next multiple
 * of 8.                                                */
typedef enum {
  CUSHA_LAYOUT_SHARD_OFFSETS = 0,   /* u32[|S|+1] first padded position of shard s          */
  CUSHA_LAYOUT_SHARD_SIZES = 1,     /* u32[|S|]   real entries of shard s                   */
  CUSHA_LAYOUT_SRC_INDEX = 2,       /* u16[P]     SrcIndex - i*|N| (i = source shard; GS)    */
  CUSHA_LAYOUT_DEST_LOCAL = 3,      /* u16[P]     DestIndex - s*|N| (filler = |N|)         */
  CUSHA_LAYOUT_EDGE_ID = 4,         /* u32[P]     input edge index (filler = 0xFFFFFFFF)    */
  CUSHA_LAYOUT_WINDOWS = 5,         /* u32[(|S|+1)*|S|] win[i*|S|+j] = start of W_ij        */
  CUSHA_LAYOUT_CW_OFFSETS = 6,      /* u32[|S|+1] first padded position of CW_i             */
  CUSHA_LAYOUT_CW_SIZES = 7,        /* u32[|S|]   real entries of CW_i                      */
  CUSHA_LAYOUT_CW_SRC_LOCAL = 8,    /* u16[Q]     SrcIndex - i*|N| per padded CW entry      */
  CUSHA_LAYOUT_MAPPER = 9,          /* u32[Q]     padded shard position (filler = trash P)  */
  CUSHA_LAYOUT_OUT_DEGREE = 10,     /* u32[|V|]   out-degree (PR NbrsNum, L318)            */
  CUSHA_LAYOUT_RUN_K = 11,          /* u32[R]     CW position of each Mapper run's first entry (CUSHA_RLE builds) */
  CUSHA_LAYOUT_RUN_T = 12,          /* u32[R]     its Mapper target; one run per non-empty W_ij      */
  CUSHA_LAYOUT_CW_WINDOW = 13,      /* u16[Q]     j of the window W_ij holding each CW_i entry (filler 0xFFFF) */
  CUSHA_LAYOUT_CW_DELTA = 14,       /* u32[|S|*|S|] Mapper in window form: Mapper[k] = delta[i*|S|+j] + k
                                                  (mod 2^32) for every real entry k of CW_i in W_ij  */
  CUSHA_LAYOUT_CW_PARTITION_OFFSETS = 15 /* partitioned only: u32[Sl*(G+1)]: CW_i's entries aimed at
                                                  partition q are [p[il*(G+1)+q], p[il*(G+1)+q+1])   */
} cusha_layout_part;
/* Returns the element count of `part` in *count (bytes = count * element size);
 * copies it to `out` (host) when out != NULL and out_bytes is large enough.
 * Parts not held by the representation (or released after the build, see
 * keep_layout) return CUSHA_EUNSUPPORTED.  Unpartitioned graphs only.      */
CUSHA_API int cusha_get_layout(const cusha_graph* g, cusha_layout_part part, void* out, size_t out_bytes, uint64_t* count);

/* The same for partition `p` of a partitioned graph (row e): p < G in the
 * one-process simulation, p = 0 (this rank's) with one process per GPU.
 * Sizes are the partition's: Sl = its shards, positions local to it; the
 * Mapper holds positions in the OWNING partition's SrcValue; OUT_DEGREE and
 * the window rows cover its own vertices / source shards.                  */
CUSHA_API int cusha_get_part_layout(const cusha_graph* g, uint32_t p, cusha_layout_part part, void* out,
                                    size_t out_bytes, uint64_t* count);

/* Statistics of partition p (as cusha_get_stats, with device_bytes,
 * entries_padded and the last run's byte / edge counts of that partition). */
CUSHA_API int cusha_get_part_stats(const cusha_graph* g, uint32_t p, cusha_stats* s);

/* Return the unused blocks of the library's private device-memory pool on
 * `device` to the driver.  Freed graphs keep their memory in that pool (so
 * repeated builds do not map HBM again); it is never shared with torch or
 * NCCL.  Errors: CUSHA_ECUDA.                                              */
CUSHA_API int cusha_trim_memory(int device);

/* Diagnostic timeline (tools/timeline.py): only a library built with
 * -DCUSHA_TIMELINE=1 records it; the product build returns CUSHA_EUNSUPPORTED.
 * Copies up to out_bytes of the per-ticket %globaltimer stamps of the last
 * overlapped-pass run into `out` (host): 10 u32 words per ticket
 * (ticket = pass * |S| + shard; word meaning in csrc/kernels.cu, kTlSlots).
 * Returns the number of tickets copied (>= 0) or a negative error code.    */
CUSHA_API int cusha_diag_timeline(void* out, size_t out_bytes);

/* ---------------------------------------------------------- host logic */
/*
 * The shard-size rule of L310 (§4 "Selecting shard size"), pure host code:
 * |N|0 = the |N| making the average window |E||N|^2/|V|^2 (L173) equal 32
 * (warp size), then snapped to the nearest of the sizes that use a whole
 * share of the SM's shared memory, N_k = floor((smem_per_sm/k - reserved)/
 * vertex_bytes) for k = 1..32 resident blocks, capped at 65534 and at |V|.
 * smem_per_sm = 0 selects B200's 233472 bytes per SM with reserved_per_block =
 * 1024 (the value passed is then ignored); otherwise both are taken as given
 * (e.g. 49152 / 0 reproduces L310's 48 KB examples: 6K at 2 blocks, 3K at 4).
 */
CUSHA_API uint32_t cusha_shard_size(uint32_t num_vertices, uint64_t num_edges, uint32_t vertex_bytes, uint32_t smem_per_sm,
                          uint32_t reserved_per_block);

/* Bytes per vertex of cusha_get_values for alg (4 or 8), 0 if invalid. */
CUSHA_API size_t cusha_value_bytes(cusha_algorithm alg);

/* Thread-local message for the last failing call on this thread ("" if none). */
CUSHA_API const char* cusha_last_error(void);

/* CUSHA_ABI_VERSION of the loaded library. */
CUSHA_API int cusha_abi_version(void);

/* One process per GPU (world_size > 1 with a rank): this rank's CUDA IPC
 * handles (CUSHA_IPC_BLOB_BYTES, host buffer).  Errors: CUSHA_ESTATE (not a
 * one-process-per-GPU graph), CUSHA_EINVAL, CUSHA_ECUDA.                    */
CUSHA_API int cusha_ipc_export(cusha_graph* g, void* out, size_t bytes);

/* Transport IPC: map every other rank's arrays; `all` holds world_size blobs
 * from cusha_ipc_export in rank order (bytes = world_size *
 * CUSHA_IPC_BLOB_BYTES).  Required once before the first cusha_run.
 * cusha_run and cusha_get_values are collective: every rank calls them in the
 * same order.  Errors: CUSHA_ESTATE, CUSHA_EINVAL, CUSHA_ECUDA.             */
CUSHA_API int cusha_ipc_connect(cusha_graph* g, const void* all, size_t bytes);

/* Multi-GPU helper: write a fresh 128-byte ncclUniqueId to out128 (rank 0
 * calls this and broadcasts it, e.g. over torch.distributed).  NCCL
 * (libnccl.so.2) is loaded at run time; CUSHA_EUNSUPPORTED if absent. */
CUSHA_API int cusha_nccl_unique_id(void* out128);

/* Host logic of the destination-range partition (pure host, no device):
 * split shards 0..num_shards-1 into `parts` contiguous ranges of near-equal
 * total work[s] (cusha_build_graph uses stage-2 + stage-4 entries per shard).
 * bounds[parts+1] receives 0 = b0 <= b1 <= ... <= b_parts = num_shards; range
 * q = [b_q, b_{q+1}).  Deterministic: every rank computes the same bounds. */
CUSHA_API int cusha_partition_shards(uint32_t num_shards, const uint64_t* work, uint32_t parts, uint32_t* bounds);

/* The partition a graph was built with: writes G+1 bounds (G = 1 for an
 * unpartitioned graph) to bounds (host, cap entries); returns G. */
CUSHA_API int cusha_get_partition(const cusha_graph* g, uint32_t* bounds, uint32_t cap);

#ifdef __cplusplus
}
#endif
#endif /* CUSHA_H */
