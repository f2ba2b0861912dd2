/*
 * dfg.h -- C ABI of the B200-native derived-field generator (libdfg.so).
 *
 * The method (Harrison et al., SC-companion 2012; /root/reference/PAPER.md,
 * cited as L<n>): a host application hands the framework an expression
 * written in a VisIt-style language plus its input arrays and gets the
 * derived field back, in situ (L116-L118).  The expression is parsed into a
 * dataflow network (L66-L76), initialised (topological order, reference
 * counts, L85) and executed by one of three strategies built from one
 * library of primitives (L86-L105): roundtrip, staged or fusion.  The
 * network is built once and re-executed whenever the data change (L122).
 *
 * Conventions for every entry point:
 *   - returns DFG_OK (0) or a negative dfg_status; dfg_last_error() gives a
 *     thread-local message for the last failing call of this thread;
 *   - no entry point falls back to the CPU: without a usable CUDA device the
 *     device-touching calls return DFG_E_CUDA;
 *   - sizes are int64 element counts unless the name says bytes;
 *   - fields are cell-centred (L154, L223), x fastest:
 *       value(i, j, k) = field[i + nx * (j + ny * k_local)]
 *     scalar arrays are T[nz][ny][nx]; vector results (grad3d, compose) are
 *     stored 4-wide, T[nz][ny][nx][4] (the OpenCL vector types of L104),
 *     unused lanes 0;
 *   - T is float (DFG_F32) or double (DFG_F64), fixed per mesh.
 */
#ifndef DFG_H
#define DFG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dfg_mesh_s* dfg_mesh;
typedef struct dfg_plan_s* dfg_plan;

/* Execution strategies, L88-L105. */
typedef enum {
  DFG_ROUNDTRIP = 0, /* one kernel per primitive, every result to the host (L92) */
  DFG_STAGED = 1,    /* one kernel per primitive, intermediates on the device (L96); with the
                        inputs and the output on the device the first execute for a binding
                        is captured into a CUDA graph (kernels + stream-ordered allocations
                        and frees) that later executes replay while the output and input
                        pointers stay the same (environment DFG_GRAPH=0: plain launches) */
  DFG_FUSED = 2,     /* one generated kernel, intermediates in registers (L97) */
  DFG_STREAMED = 3,  /* fusion over z-chunks streamed through a 3-slot device ring with
                        overlapped upload / kernel / download (the paper's future-work
                        streaming strategy, L245 / L344); bounded device memory, so host
                        meshes larger than HBM work; single slab; with everything
                        device-resident it is DFG_FUSED.  Chunk height: ~512 MiB of
                        input per chunk (env DFG_STREAM_PLANES overrides); each field
                        plane crosses PCIe once (chunk halos are copied on the device).
                        Pinned host buffers are needed for the copies to overlap. */
  DFG_REFERENCE = 4, /* the hand-written reference kernel of a quantity (L243): expr is
                        "velmag", "vortmag" or "qcrit" (fields u, v, w must be bound);
                        same I/O and TMA pipeline as fusion, fewer flops (derivative =
                        numerator x reciprocal spacing, FMA, Q = -1/2 tr(J^2)); agrees
                        with the network within floating-point tolerance, not bitwise */
  DFG_HYBRID = 5     /* staged execution (the same kernels and results) that fits a
                        dev_mem_cap below the staged footprint by spilling
                        intermediates to pinned host memory (SURVEY 8f NEXT #3,
                        the Fig. 2 argument L107-L114): list
                        order if it fits the cap, else the memory-aware order, and
                        if that does not fit either, before each array that does
                        not fit the resident array with the furthest next use is
                        evicted (an intermediate is copied to the host once, an
                        uploaded input is dropped) and brought back when needed.
                        All inputs and the output either in host memory (the
                        paper's host interface) or all on the device; whole mesh
                        only.  DFG_E_NOMEM at compile if the cap is below some
                        filter's working set (its operands plus its result, plus
                        the resident inputs and output in device mode). */
} dfg_strategy;

typedef enum { DFG_F32 = 0, DFG_F64 = 1 } dfg_dtype;

typedef enum {
  DFG_OK = 0,
  DFG_E_INVALID = -1,     /* bad argument (null handle, size, coordinates, name) */
  DFG_E_PARSE = -2,       /* expression syntax; message carries line:col      */
  DFG_E_UNDEFINED = -3,   /* unknown identifier or function                   */
  DFG_E_TYPE = -4,        /* arity, scalar/vector mismatch, index out of range */
  DFG_E_NOMEM = -5,       /* footprint above the cap, or device allocation failed (L309) */
  DFG_E_NVRTC = -6,       /* fused-kernel compilation failed                  */
  DFG_E_CUDA = -7,        /* CUDA runtime/driver error or no device            */
  DFG_E_NCCL = -8,        /* NCCL unavailable or failed                        */
  DFG_E_UNBOUND = -9,     /* an input the network reads has no bound buffer    */
  DFG_E_UNSUPPORTED = -10,/* valid request this build does not implement       */
  DFG_E_RANGE = -11       /* caller buffer too small (see *needed)             */
} dfg_status;

/* Device events and memory of a plan (Table II L271-L285 quantities and the
 * Fig. 6 high-water mark, L245-L247).  Counters accumulate over executes
 * until dfg_reset_stats(). */
typedef struct {
  int64_t executes;
  int64_t h2d_count;            /* host->device transfers ("Dev-W")           */
  int64_t d2h_count;            /* device->host transfers ("Dev-R")           */
  int64_t kernel_count;         /* kernel executions ("K-Exe")                */
  int64_t h2d_bytes;
  int64_t d2h_bytes;
  int64_t halo_bytes;           /* bytes received into ghost planes, or read
                                   from the neighbours' planes (peer halo)    */
  int64_t dev_highwater_bytes;  /* max live problem-sized device arrays, incl.
                                   bound device inputs and the output (Fig. 2) */
  int64_t predicted_highwater_bytes; /* model of the last-executed mode        */
  int64_t predicted_hbm_bytes;  /* algorithmic device bytes of one execute    */
  int64_t predicted_pcie_bytes; /* algorithmic host<->device bytes of one execute */
  double last_ms;               /* device time of the last execute (CUDA events);
                                   waits for it to finish; -1 if none          */
  double kernel_ms_sum;         /* device time of every fused-kernel launch since
                                   the last reset (CUDA events around the launch
                                   on the execute stream; no host sync inside
                                   execute -- resolved when stats are read)      */
  int64_t kernel_launches_timed;/* launches summed in kernel_ms_sum            */
} dfg_stats;

/* ---------------------------------------------------------------- version */
int dfg_version(void);                 /* 100 * major + minor */
const char* dfg_last_error(void);      /* never NULL; "" after success */

/* ------------------------------------------------------------------- mesh
 * Rectilinear mesh (L86, L165): nx x ny x nz cells; point coordinates
 *   x[0..nx], y[0..ny], z[0..nz_global]  (host pointers, element type T,
 *   strictly increasing, finite) -- copied, the caller keeps ownership.
 * z-slab decomposition (ghost data, L255 / L315): this mesh object holds
 *   the cells k in [z_offset, z_offset + nz_local) of a global mesh with
 *   nz_global cells in z; ghost = 0 or 1 extra planes on both ends of every
 *   bound field buffer (filled by the halo exchange of dfg_execute).
 *   Single GPU: nz_local = nz_global, z_offset = 0, ghost = 0.
 * The mesh is created on the CUDA device current at the call; it builds and
 * uploads the per-axis spacing tables (R1).
 * Errors: DFG_E_INVALID (sizes < 1, z range outside the global mesh,
 * coordinates not strictly increasing or not finite, ghost not 0/1),
 * DFG_E_CUDA (no device). */
int dfg_create_mesh(dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz_local,
                    const void* x, const void* y, const void* z,
                    int64_t nz_global, int64_t z_offset, int ghost,
                    dfg_mesh* out);
/* VisIt-style sub-grid (the paper's distributed run: 3072 sub-grids of
 * 192 x 192 x 256 cells "plus the necessary ghost cells", L253-L255, L315;
 * SURVEY 8f NEXT #4): local nx x ny x nz cells at offsets (i0, j0, k0) of a
 * global NX x NY x NZ mesh whose point coordinates x[0..NX], y[0..NY],
 * z[0..NZ] are given (host, T).  ghost = 1: every bound field buffer carries
 * a one-cell ghost shell on all six faces, T[nz+2][ny+2][nx+2], filled by
 * the CALLER (VisIt's ghost exchange) -- no halo transport is used; cells on
 * the global mesh boundary ignore their ghost cells (one-sided differences,
 * reading R1).  ghost = 0 only for the whole mesh.  Output: T[nz][ny][nx].
 * Row layout (like cudaMallocPitch): a buffer is T[nz+2][ny+2][row_pitch];
 * in each row the owned cells sit at columns x_offset .. x_offset+nx-1, the
 * ghost columns at x_offset-1 and x_offset+nx, anything else is padding that
 * is never read.  x_offset = 0 means ghost, row_pitch = 0 means
 * x_offset + nx + ghost (the packed shell).  Fusion (and reference)
 * strategies only; the TMA fast path needs nx, x_offset and row_pitch times
 * sizeof(T) to be multiples of 16 bytes (TMA box coordinates along a row
 * must be 16-byte aligned) -- e.g. for the paper's 192-wide fp32 blocks
 * x_offset 4, row_pitch 200; other layouts use the general kernel.
 * Errors as dfg_create_mesh; DFG_E_INVALID unless ghost <= x_offset and
 * x_offset + nx + ghost <= row_pitch. */
int dfg_create_block(dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz,
                     const void* x, const void* y, const void* z,
                     int64_t NX, int64_t NY, int64_t NZ,
                     int64_t i0, int64_t j0, int64_t k0, int ghost,
                     int64_t row_pitch, int64_t x_offset, dfg_mesh* out);

/* Idempotent on NULL.  Plans keep what they need alive: destroying a mesh
 * with live plans is allowed (the plans stay valid). */
void dfg_destroy_mesh(dfg_mesh mesh);

/* Even z-slab split used by the driver:
 *   nz_r = nz_global / n + (rank < nz_global % n), z_offset = sum of the
 *   preceding slabs.  DFG_E_INVALID unless 1 <= nranks <= nz_global. */
int dfg_partition(int64_t nz_global, int nranks, int rank,
                  int64_t* z_offset, int64_t* nz_local);

/* Ghost-plane map of this slab, 16 int64:
 *   rank, nranks, NZ, k0, k1, nz_r, has_lo, has_hi, peer_lo, peer_hi,
 *   send_lo_local_plane, send_hi_local_plane, recv_lo_local_plane,
 *   recv_hi_local_plane, plane_bytes, halo_width
 * Local planes count the lower ghost plane as 0 (owned planes 1..nz_r);
 * absent entries are -1.  rank/nranks are 0/1 until a communicator is set. */
int dfg_halo_map(dfg_mesh mesh, int64_t out[16]);

/* Multi-GPU halo transport, one process per GPU (NCCL point-to-point,
 * L255 ghost exchange re-done over NVLink).  dfg_nccl_unique_id fills 128
 * bytes on rank 0; the caller broadcasts them (torch.distributed) and every
 * rank calls dfg_mesh_init_comm on the device that owns its mesh.
 * NCCL is loaded at run time (libnccl.so.2); DFG_E_NCCL if unavailable. */
int dfg_nccl_unique_id(void* out128);
int dfg_mesh_init_comm(dfg_mesh mesh, const void* id128, int rank, int nranks);

/* Peer-memory halo, one process per GPU (the B200 path for z-slabs: the
 * fused kernel reads the neighbours' boundary planes in place over NVLink
 * instead of receiving copies).
 *
 * dfg_mesh_peer_export writes DFG_PEER_BLOB_BYTES bytes describing the slab:
 * CUDA IPC handles (and offsets) of every field bound with on_device = 1 and
 * of a small flag block the library allocates, the slab's extent and type.
 * Bind the fields first; rebinding a field afterwards makes dfg_execute fail
 * with DFG_E_INVALID until the blob is exported and linked again.  The fields
 * must be cudaMalloc-backed (IPC), the mesh a z-slab with ghost = 1.
 *
 * Every rank exchanges blobs (e.g. torch.distributed all_gather_object) and
 * calls dfg_mesh_link_peers with the blob of the slab directly below (lo,
 * NULL on rank 0) and directly above (hi, NULL on the last rank).  Checks:
 * magic, type, plane size, global depth and adjacency (DFG_E_INVALID);
 * DFG_E_UNSUPPORTED if CUDA IPC is refused (then neither side is linked).
 * Both blobs NULL unlinks (the slab falls back to NCCL / local links).  The
 * mappings stay open until the mesh is destroyed (the exporting ranks must
 * keep their fields alive).
 *
 * A linked slab's dfg_execute (fused / reference strategies) orders itself
 * with its neighbours by step flags (stream memory operations: the execute
 * publishes "ready", waits for the neighbours' "ready" before the boundary
 * planes, and before returning the stream waits until both neighbours have
 * read its planes), so every rank must execute the same sequence of plans on
 * the mesh.  Its ghost planes are not written (TMA reads the neighbours'
 * buffers), except for layouts the TMA kernel cannot take, which copy the two
 * planes through the mappings first.  The output must be on the device. */
#define DFG_PEER_BLOB_BYTES 4096
int dfg_mesh_peer_export(dfg_mesh mesh, void* blob, size_t cap);
int dfg_mesh_link_peers(dfg_mesh mesh, const void* lo_blob, const void* hi_blob);

/* Probe of the in-place transport before a link:
 * opens the flag allocation of the slab that exported `blob` (host pointer,
 * DFG_PEER_BLOB_BYTES) through CUDA IPC on the CURRENT device, reads its
 * 8 KiB probe block (a pattern the exporter wrote) with one TMA load through
 * a tensor map over the mapping -- the access the boundary-plane launches
 * make -- and sets *ok = 1 if every word matches, 0 otherwise; the mapping
 * is closed again.  Run it in a separate short-lived process (bench.py does):
 * the caller of dfg_mesh_link_peers must not be the process a faulting
 * transport takes down.  The exporter must keep its mesh alive meanwhile.
 * Errors: DFG_E_INVALID (null argument, not an export blob),
 * DFG_E_UNSUPPORTED (IPC refused), DFG_E_CUDA. */
int dfg_peer_probe(const void* blob, int* ok);

/* Single-process halo transport: slabs that live in one process (one or
 * several devices) exchange ghost planes with device-to-device copies.
 * `lo` must hold the slab directly below `hi` (lo.k1 == hi.k0). */
int dfg_mesh_link_local(dfg_mesh lo, dfg_mesh hi);

/* ----------------------------------------------------------------- fields
 * Bind a cell-centred scalar input under `name` (an identifier; not a
 * keyword, not dims/x/y/z, not f<digits>).  BORROWED: the buffer must stay
 * valid and unchanged in shape until the executes that read it complete.
 * Layout T[nz_local + 2*ghost][ny][nx] (ghost planes at both ends).
 * on_device = 1: a CUDA pointer on the mesh's device (in situ mode);
 * on_device = 0: a host pointer -- the paper's host interface (L118):
 * the strategies upload it and count the transfers (Table II).  Host
 * pointers are single-slab only (nranks = 1).  Rebinding replaces;
 * ptr = NULL unbinds.  The fused kernel's TMA fast path additionally wants
 * 16-byte aligned device pointers and nx*sizeof(T) % 16 == 0; other
 * layouts run the general kernel with the same arithmetic. */
int dfg_bind_field(dfg_mesh mesh, const char* name, void* ptr, int on_device);

/* ------------------------------------------------------------------ plans
 * Parse -> dataflow network -> plan (L64-L105).  Every identifier the
 * program reads must be a field bound at this point, an earlier assignment
 * target, or one of dims/x/y/z as grad3d arguments.
 * dev_mem_cap: bytes of problem-sized device arrays the plan may hold at
 * once (0 = unlimited); checked against the predicted footprint here
 * (DFG_E_NOMEM) and against the live ledger during execute.
 * Fused plans generate, NVRTC-compile (sm_100a) and load their kernel here.
 * Errors: DFG_E_PARSE, DFG_E_UNDEFINED, DFG_E_TYPE, DFG_E_NOMEM,
 * DFG_E_NVRTC, DFG_E_CUDA, DFG_E_UNSUPPORTED (staged/roundtrip on a
 * multi-slab mesh). */
int dfg_compile(dfg_mesh mesh, const char* expr, dfg_strategy strategy,
                size_t dev_mem_cap, dfg_plan* out);
void dfg_destroy_plan(dfg_plan plan);

/* Execute on `cuda_stream` (cudaStream_t; NULL = legacy default stream).
 * out: T[nz_local][ny][nx] (or [..][4] for a vector program), a device
 * pointer if out_on_device else a host pointer.  Fused and staged enqueue
 * asynchronously when everything is on the device; any host buffer makes
 * the call synchronous (roundtrip always is).  Multi-slab meshes first
 * exchange the ghost planes of the fields grad3d reads (this writes the
 * ghost planes of the caller's buffers).
 * Errors: DFG_E_UNBOUND, DFG_E_NOMEM (ledger cap or allocation failure:
 * the paper's failed GPU cases, L309), DFG_E_CUDA, DFG_E_NCCL. */
int dfg_execute(dfg_plan plan, void* out, int out_on_device, void* cuda_stream);

/* Several fused plans of ONE network on different meshes of the same device
 * -- the paper's VisIt sub-grids, 12 per GPU (L253-L255, L315) -- in one
 * launch: the persistent TMA kernel walks the concatenated tiles of all
 * meshes, so small blocks do not pay one kernel's fill and drain each.
 * outs[b]: device output of plans[b].  Used when every plan is DFG_FUSED
 * with the same generated kernel (same expression, dtype and global mesh),
 * every input device-resident and no halo exchange needed (whole meshes or
 * blocks with ghost shells): the TMA kernel when every layout is
 * TMA-eligible (see dfg_create_block), else the same pipeline with the ring
 * filled by cp.async (packed ghost shells, rows that are not 16-byte
 * multiples); otherwise the plans execute one after the other.
 * Results equal dfg_execute's bit for bit.  Stats: executes +1 on every
 * plan; the launch and its timing are counted on plans[0].
 * Errors as dfg_execute; DFG_E_INVALID for n < 1 or null entries. */
int dfg_execute_blocks(dfg_plan const* plans, int n, void* const* outs, void* cuda_stream);

int dfg_plan_stats(dfg_plan plan, dfg_stats* out);
int dfg_reset_stats(dfg_plan plan);

/* CUDA-event timing of later executes of `plan` (default 1):
 *   0  no events: last_ms stays at its previous value (-1 after a reset) and
 *      the kernel timings do not advance -- the cheapest execute;
 *   1  one event pair around each execute (stats.last_ms);
 *   2  as 1, plus one event pair around every fused-kernel launch
 *      (stats.kernel_ms_sum / kernel_launches_timed).
 * Every timestamped event costs GPU time of its own (measured ~2 us on B200),
 * which only small meshes notice.  Pending kernel timings are folded into the
 * stats first.  Errors: DFG_E_INVALID (null plan, level outside 0..2). */
int dfg_plan_set_timing(dfg_plan plan, int level);

/* Plan description: out[0] = strategy, out[1] = result width (1 or 4),
 * out[2] = number of filters, out[3] = fused kernel variant of the last
 * execute (0 none, 1 TMA pipeline, 2 general, 3 point-wise, 4 TMA
 * multi-block via dfg_execute_blocks, 5 tile: the TMA kernel's ring filled
 * by cp.async, for layouts a tensor map cannot describe, 6 tile multi-block,
 * 7 row-class kernel: rows loaded as two-plane TMA boxes per 16-byte row
 * class, x ends of reading R1 by a fixup warp -- packed ghost shells and rows
 * that are not 16-byte multiples, with 16-byte aligned bases and plane
 * strides, 8 row-class multi-block), out[4] = registers per thread of the
 * fused kernel (0 if none), out[5] = local memory per thread of that kernel
 * (bytes; spills and stack), out[6] = predicted
 * device footprint in bytes for device-resident inputs,
 * out[7] = same for host inputs, out[8] = grad3d quotient form of the fused
 * kernel, bit a set = axis a uses the two-operation exact quotient (fp32,
 * every divisor of the axis verified at mesh creation),
 * clear = the three-operation correction (or IEEE / fast division when
 * DFG_FUSED_VARIANT selects them), out[9] = tile rows per consumer warp of
 * the TMA kernel (1, 2 or 4; 0 without one), out[10] / out[11] = its tile
 * width (cells along x) / height (rows along y), out[12] = z-chunk length
 * (planes per work item) of the last TMA launch (0 before one), out[13] =
 * halo transport of the last execute (0 none, 1 NCCL, 2 local device copies,
 * 3 peer memory read in place by the kernel, 4 peer memory copied into the
 * ghost planes).  `out` must hold 14 entries. */
int dfg_plan_info(dfg_plan plan, int64_t out[14]);

/* Arithmetic of a plan and the inputs on which its results equal the
 * oracle's (the literal network evaluated in T, reading R6; DESIGN.md
 * section 5): out[0] = grad3d quotient (0 IEEE div.rn, 1 exact in the
 * normal range: two-operation / Markstein with the reciprocal tables,
 * 2 fast num * (1/d)), out[1] = 1 if power-of-two scale folding rewrites
 * the fused body, out[2] = two-operation axes mask (out[0] == 1),
 * out[3] = exactness domain: 2 = bit-identical for EVERY input (IEEE
 * operations only: the staged / roundtrip / hybrid kernels, and
 * DFG_FUSED_VARIANT=ieee), 1 = bit-identical on the cells where every
 * input, every grad3d numerator and every value of the literal network is 0
 * or normal with 2^p of headroom (and no numerator is -0: DESIGN.md
 * section 5; the default fused kernel),
 * 0 = within tolerance only (fast quotient, hand-written reference
 * bodies).  `out` must hold 4 entries.  Host only; no device work. */
int dfg_plan_arith(dfg_plan plan, int64_t out[4]);

/* Execution order of the plan's filters (ids of the canonical text).  Staged
 * plans run the paper's list order unless a dev_mem_cap rejected it and the
 * memory-aware order (greedy minimum live memory) fits --
 * or DFG_STAGED_ORDER=greedy was set at compile.  Writes min(cap, n) ids;
 * *n = number of filters. */
int dfg_plan_schedule(dfg_plan plan, int32_t* order, size_t cap, size_t* n);

/* Transfer schedule of a DFG_HYBRID plan for the binding mode of its last
 * execute (or, before the first, of the bindings at compile): n events, each
 * two int32 (kind, ref), kinds: 0 upload input, 1 reload intermediate from
 * its host copy, 2 spill intermediate to the host, 3 discard a device copy
 * whose host copy is valid, 4 drop an uploaded input, 5 run filter, 6 sink
 * device -> host, 7 sink from the host copy (no transfer), 8 sink host copy
 * -> device output.  ref = filter id, or -1 - (input index) for a bound
 * input.  Writes min(cap, n) events (2 int32 each); *n = number of events.
 * DFG_E_INVALID for other strategies. */
int dfg_plan_transfers(dfg_plan plan, int32_t* events, size_t cap, size_t* n);

/* Canonical network text (R10) -- stands in for the paper's
 * optional Python script of network-definition API calls (L84).
 * Copies up to cap bytes incl. the NUL; *needed = full size incl. NUL;
 * DFG_E_RANGE if cap is too small. */
int dfg_dump_dag(dfg_plan plan, char* buf, size_t cap, size_t* needed);
/* Generated CUDA source of a fused plan (the paper's dynamic kernel
 * generator output, L97-L105); same buffer protocol. */
int dfg_dump_kernel(dfg_plan plan, char* buf, size_t cap, size_t* needed);

/* ------------------------------------------------------- host-only tools
 * Need no GPU: the parser / network builder, the strategy model and the
 * kernel generator on their own, for tests and tooling. */

/* Paper-layout compatibility (Table I): the
 * paper's data carry point coordinates as full 3-D arrays x3, y3, z3 of shape
 * [nz+1][ny+1][nx+1] (x fastest, type T).  Extracts the per-axis point arrays
 * x[nx+1], y[ny+1], z[nz+1] for dfg_create_mesh and checks that the mesh is
 * rectilinear (x3 depends on i only, y3 on j only, z3 on k only; bitwise):
 * DFG_E_INVALID otherwise.  Host pointers; no device needed. */
int dfg_points3d_to_axes(dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz,
                         const void* x3, const void* y3, const void* z3,
                         void* x, void* y, void* z);

/* Parse + lower `expr` with the named scalar inputs; write the canonical
 * text.  Same errors as dfg_compile's language errors. */
int dfg_dag_dump(const char* expr, const char* const* inputs, int n_inputs,
                 dfg_dtype dtype, char* buf, size_t cap, size_t* needed);

/* Planner's predictions for one execute: out[0..2] = h2d, d2h, kernels;
 * out[3] = footprint in problem-array units (scalar 1, vector 4).
 * host_mode = 1: inputs and output in host memory (Table II, Fig. 2);
 * 0: everything device resident. */
int dfg_model(const char* expr, const char* const* inputs, int n_inputs,
              dfg_strategy strategy, int host_mode, int64_t out[4]);

/* The DFG_HYBRID planner on its own: schedule of
 * `expr` in host (host_mode = 1) or device mode under cap_units problem
 * arrays, filters in `order` (n_order ids, a topological order; NULL = list
 * order).  Events as dfg_plan_transfers (min(cap, n) written, *n = count);
 * out[0..4] = high-water units, h2d transfers, d2h transfers, h2d units,
 * d2h units.  DFG_E_NOMEM if the cap is below a filter's working set,
 * DFG_E_INVALID if `order` is not a topological order. */
int dfg_hybrid_model(const char* expr, const char* const* inputs, int n_inputs,
                     int host_mode, int64_t cap_units, const int32_t* order, size_t n_order,
                     int32_t* events, size_t cap, size_t* n, int64_t out[5]);

/* Generate the fused kernel source for `expr` on an nx x ny x nz mesh and,
 * if compile != 0, NVRTC-compile it for sm_100a (no device needed); on
 * success *regs / *spill (may be NULL) get the ptxas figures of the TMA
 * kernel.  Sources use the two-operation quotient on every axis (the
 * kernel of a mesh whose divisors all verified) unless the environment sets
 * DFG_FUSED_VARIANT=markstein.  Writes the source with the buffer protocol
 * above. */
int dfg_fused_source(const char* expr, const char* const* inputs, int n_inputs,
                     dfg_dtype dtype, int64_t nx, int64_t ny, int64_t nz,
                     int compile, char* buf, size_t cap, size_t* needed,
                     int* regs, int* spill);

/* The paper's programs as text, for callers: "velmag", "vortmag", "qcrit"
 * (Fig. 3; Q completed per DESIGN.md readings G1-G3; inputs u,
 * v, w) and "intro" (L19; inputs b, c).  Buffer protocol as dfg_dump_dag:
 * *needed = bytes incl. the terminating NUL; DFG_E_RANGE if cap is too
 * small; DFG_E_INVALID for an unknown name.  Host only. */
int dfg_paper_program(const char* which, char* buf, size_t cap, size_t* needed);

/* Two-operation quotient check, exposed for tests (DESIGN.md section 5,
 * csrc/div2.hpp).  A fused kernel forms a grad3d derivative num / d (L99,
 * reading R1) as RN(num*r + RN(num*yl)) with r = RN(1/d), yl = RN(1/d - r)
 * on every axis whose divisors all pass this check, else with Markstein's
 * three-operation correction.  For each of the n divisors d[i] (host array
 * of T = dtype; positive normal numbers, else DFG_E_INVALID) the library
 * forms r and yl as the spacing tables do and sets ok[i] = 1 if the scheme
 * equals RN(num / d) for every numerator in the normal range:
 *   method 0: certification by candidate numerators (fp32 and fp64; the
 *             handful of numerators whose quotient lies within the scheme's
 *             error bound of a rounding boundary; what fp64 meshes use);
 *   method 1: exhaustive, all 2^23 fp32 significands on the host (fp32
 *             only, else DFG_E_UNSUPPORTED; ~10 ms per divisor; fp32 meshes
 *             run the same enumeration on the device).
 * tested (may be NULL): candidate numerators evaluated per divisor (method 0;
 * 0 for method 1).  Host only, no device needed; caller owns all arrays. */
int dfg_div2_check(dfg_dtype dtype, const void* d, int64_t n, int method, uint8_t* ok, int64_t* tested);

#ifdef __cplusplus
}
#endif
#endif /* DFG_H */
