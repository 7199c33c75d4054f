/*
 * somier.h -- the Somier time step spread over devices: C ABI of libsomier.so.
 *
 * Paper (§V "Use case: Somier mini-app", 319-344):
 * a 3-D grid of springs; each time step runs the kernels forces (a stencil over
 * the neighbour cells), accelerations, velocities, positions, and a "centers"
 * reduction over the positions. Four variables x three
 * 3-D fp64 grids. The step is spread over devices along the
 * outermost dimension with halos "between chunks in the outermost dimension"
 * (PAPER.md:328), i.e. `target spread` over the i-loop with
 * map(to: X[omp_spread_start-1 : omp_spread_size+2]).
 * Where the paper is silent the readings of DESIGN.md §3
 * apply: central Hooke springs to the 6 face neighbours, six fixed faces,
 * semi-implicit Euler with double-buffered (Jacobi) positions, centre of mass
 * over all nodes by an exact int128 fixed-point sum, vmax = max |v|.
 *
 * One call of somier_step = the paper's five kernels fused into ONE sm_100a
 * kernel launch per chunk (K1_TB2: per two steps); the halo exchange is fused
 * into the same kernel by default (boundary planes are stored straight into
 * the neighbour chunk's halo slot, through NVLink P2P / CUDA IPC when the
 * neighbour is on another GPU; somier_params.exchange selects the unfused copy
 * or NCCL routes instead).
 *
 * Lifetime (mirrors the data directives):
 *   somier_init        ~ target enter data spread map(to: X[start-1:size+2], V[start:size])
 *   somier_load        ~ target update spread to(...)           (host -> device)
 *   somier_step        ~ target spread teams distribute parallel for ... nowait
 *   somier_sync        ~ taskgroup / taskwait
 *   somier_stats       ~ the "centers" result of the last completed step
 *   somier_stats_history ~ the "centers" of every step (the last 126)
 *   somier_read        ~ target exit data spread map(from: X[start:size], V[start:size])
 *   somier_destroy     ~ end of the data region
 *
 * Conventions: every call returns spread_status (spread.h). Handles are
 * library-owned, not thread-safe (one host thread per handle). CUDA errors
 * raised by asynchronous work are sticky and reported by the next blocking
 * call (somier_sync / somier_stats / somier_read) as SPREAD_ECUDA, with the
 * CUDA message in spread_last_error(). A failed somier_init leaves no
 * allocation behind.
 */
#ifndef PAPER_SOMIER_H
#define PAPER_SOMIER_H

#include <stddef.h>
#include <stdint.h>

#include "spread.h"

#ifdef __cplusplus
extern "C" {
#endif

/* K1 implementations (all compute bit-identical results). */
typedef enum {
    SOMIER_K1_AUTO = 0,      /* the fastest measured: SOMIER_K1_TB2 when every chunk
                                has >= 3e6 nodes and the devices have room for its
                                deeper slabs, else SOMIER_K1_MARCH2
                                (somier_kernel_in_use tells which)                    */
    SOMIER_K1_DIRECT = 1,    /* one thread per node, 6 springs from global loads       */
    SOMIER_K1_MARCH = 2,     /* plane-marching, smem-staged, 3 springs/node with reuse */
    SOMIER_K1_MARCH2 = 3,    /* as MARCH with two rows per warp (32 x 16 tiles)        */
    SOMIER_K1_TB2 = 4        /* two time steps per pass over HBM (temporal blocking),
                                deep-halo exchange between chunks (every chunk >= 2
                                planes when there are several, else MARCH2); V
                                double-buffered; both steps' stats computed          */
} somier_kernel;

/* Operation order of the step's fp64 arithmetic (reading S22).
 * north_star's correctness bar: positions and velocities within a max relative
 * error of 1e-10 of the oracle after 100 steps, "FMA contraction the only
 * allowed difference", partitioned runs bit-identical to the 1-GPU run.
 *   EXACT: every operation rounded separately in the oracle's order (reading
 *          S13): the state and the stats are bit-identical to the oracle.
 *   FMA:   the spring's d.d as fma(dz, dz, fma(dy, dy, dx*dx)) and the
 *          semi-implicit Euler update as v' = fma(a, h, v), x' = fma(v', h, x)
 *          (12 fewer fp64 operations per node-update, 108 -> 96); everything
 *          else, the stats included, unchanged. Within the 1e-10 bar of the
 *          oracle, and still bit-identical across kernels, chunkings, device
 *          lists, schedules and the host-streamed mode, because every kernel
 *          evaluates a node with the same contracted expressions.          */
typedef enum {
    SOMIER_MATH_EXACT = 0,
    SOMIER_MATH_FMA = 1
} somier_math;

typedef struct {
    int64_t n[3];        /* nodes per dimension (i outermost, k contiguous); each >= 3        */
    double spacing;      /* rest-lattice spacing                                               */
    double rest_len;     /* spring rest length L                                               */
    double k_spring;     /* stiffness K                                                        */
    double mass;         /* node mass M (> 0)                                                  */
    double dt;           /* time step h (> 0)                                                  */
    double amplitude;    /* initial displacement amplitude a (|a| < rest_len / 2 recommended)  */
    uint64_t seed;       /* SplitMix64 seed of the initial displacement (reading S7)           */
    int32_t kernel;      /* somier_kernel                                                      */
    int32_t exchange;    /* somier_exchange: how boundary planes reach the neighbour chunks    */
    int32_t math;        /* somier_math: operation order of the step's fp64 arithmetic          */
    int32_t reserved;    /* must be 0                                                          */
} somier_params;

/* The halo exchange between chunks on different streams (devices / processes),
 * SURVEY.md §8(b) `overlap` and §8(e): FUSED (default) -- K1 stores its boundary
 * planes straight into the neighbours' halo slots (NVLink P2P / CUDA IPC) and
 * its boundary CTAs publish the neighbours' flags; COPY -- the unfused route for
 * A/B: K1 writes only its own slab, then the stream copies the boundary planes
 * into the neighbours' halos (cudaMemcpyAsync over P2P / IPC) and writes the
 * flags (cuStreamWriteValue64) after the whole kernel. Results are bit-identical. */
typedef enum { SOMIER_EXCHANGE_FUSED = 0, SOMIER_EXCHANGE_COPY = 1, SOMIER_EXCHANGE_NCCL = 2 } somier_exchange;
/* SOMIER_EXCHANGE_NCCL -- SURVEY.md §8(e)'s collective route: after each launch
 * the boundary planes go by ncclSend / ncclRecv (one ncclGroupStart/End per
 * launch over every chunk boundary, each list position one NCCL rank on its
 * stream; same-position boundaries are self send/recv), no flags. NCCL is
 * loaded at run time (SOMIER_NCCL_LIB, else libnccl.so.2). Single-process
 * handles create the communicators at somier_init (ncclCommInitAll; the list's
 * CUDA devices must be distinct: NCCL places one rank per GPU -- ENOTSUP
 * otherwise); multi-process handles call somier_nccl_connect with an id from
 * somier_nccl_unique_id shared by all ranks (rank = list position). */
/* (somier_nccl_unique_id / somier_nccl_connect: below, after somier_ipc_connect) */

/* Stats of one step ("centers"). The exact partial sums are
 * exported so that per-process partials can be combined exactly. */
typedef struct {
    int64_t step;         /* number of completed steps                                     */
    double centre[3];     /* (1/N) * sum over all N = n0*n1*n2 nodes of x_{t} (exact sum)  */
    double vmax;          /* sqrt(max over nodes of v.v)                                    */
    uint64_t sum_lo[3];   /* sum of round_half_even(x * 2^60), int128 two's complement, lo */
    int64_t sum_hi[3];    /* ... hi                                                         */
    uint64_t vmax2_bits;  /* IEEE-754 bits of max v.v (uint64 order == double order, >= 0)  */
    int64_t nodes;        /* number of nodes covered by these sums                          */
} somier_stats_t;

typedef struct somier_s* somier_t;

/*
 * somier_init -- single-process mode (the paper's model: one host program drives
 * every device of the list). Allocates every chunk of `s` on its device, generates
 * the initial state on the devices (reading S7; bit-identical to the oracle's),
 * enables peer access between list devices that hold neighbouring chunks.
 *   s   spread over the i-range; must be exactly range(1 : n0-2), i.e. the loop
 *       for(i=1; i<n0-1; i++) (coherence is checked, unlike the paper).
 *       The descriptor is copied; `s` may be destroyed afterwards.
 *   p   parameters (copied).
 * Errors: EINVAL (params, range mismatch, chunk too thin: every chunk must own >= 1
 * plane), ENODEV (device id >= cudaGetDeviceCount), ENOMEM, ECUDA.
 */
spread_status somier_init(spread_t s, const somier_params* p, somier_t* out);

/*
 * somier_init_on -- somier_init with the list's device ids read as LOGICAL
 * devices: list position q runs on CUDA device cuda_devices[q] (NULL = the
 * ids themselves). Several positions may share one GPU; each position keeps
 * its own stream and the cross-position protocol (in-kernel halo stores +
 * completion flags + stream waits) runs exactly as between GPUs -- how the
 * multi-device path is exercised on a one-GPU machine.
 */
spread_status somier_init_on(spread_t s, const somier_params* p, const int* cuda_devices, somier_t* out);

/*
 * somier_init_local -- multi-process mode (one process per GPU): this handle owns
 * only the chunks at list position `device_pos` of `s`, on CUDA device
 * `cuda_device` of this process (-1: the id the list gives for that position;
 * pass the local ordinal when each process sees its GPU under another index,
 * e.g. with CUDA_VISIBLE_DEVICES). Chunks owned by other processes are reached
 * after somier_ipc_export / somier_ipc_connect; until then somier_step returns
 * ESTATE if a neighbour chunk is remote. somier_load is collective in this mode:
 * every process must load (and the caller must barrier) before anyone steps.
 */
spread_status somier_init_local(spread_t s, const somier_params* p, int device_pos, int cuda_device,
                                somier_t* out);

/*
 * somier_ipc_export -- serialise the CUDA IPC handles of this handle's halo slots
 * and exchange flags into buf (capacity cap bytes); *len receives the size used
 * (call with buf == NULL to query). The blob is opaque and position-independent.
 */
spread_status somier_ipc_export(somier_t h, void* buf, size_t cap, size_t* len);

/*
 * somier_ipc_connect -- import the blobs of all processes (including this one,
 * which is skipped), open the handles of the remote neighbour chunks.
 * Errors: EINVAL (malformed blob, other spread or params), ECUDA.
 */
spread_status somier_ipc_connect(somier_t h, const void* const* blobs, const size_t* lens, int nblobs);

/* SOMIER_EXCHANGE_NCCL, multi-process: one rank creates an id, every rank
 * passes it with nranks = the list length (rank = device_pos). Errors: ENOTSUP
 * (NCCL unavailable), ESTATE (not a multi-process NCCL handle), ENCCL. */
spread_status somier_nccl_unique_id(void* id_out /* 128 bytes */);
spread_status somier_nccl_connect(somier_t h, const void* id /* 128 bytes */, int nranks);

/* Enqueue nsteps >= 0 time steps on every owned chunk; returns after enqueue (nowait). */
spread_status somier_step(somier_t h, int64_t nsteps);

/* Block until all enqueued work of this handle is complete (taskgroup). */
spread_status somier_sync(somier_t h);

/*
 * somier_stats -- blocking; stats after the last completed step, combined over
 * the chunks THIS handle owns (plus the fixed end planes it holds as halos).
 * In single-process mode that is the whole grid. In multi-process mode combine
 * the per-process results with somier_stats_combine.
 * Exact-stats domain (S18): the centre sums are exact while every
 * position is finite with |x| < 2^23. Each state carries an upper bound on
 * max |x| -- exact for an initialised / loaded (or, host-streamed, mapped-in)
 * state, and (B + sqrt(vmax^2) |dt|) (1 + 2^-40) for the state a step produces
 * (computed by the last CTA of each launch: no per-node cost). A state whose
 * bound is not below 2^23 (or is NaN) reports centre[] = NaN (sum_lo / sum_hi
 * are still exported; vmax is unaffected). somier_stats_combine propagates a
 * NaN centre of any partial.
 */
spread_status somier_stats(somier_t h, somier_stats_t* out);

/*
 * somier_stats_history -- blocking; the stats of EVERY step ("centers" after
 * each time step): out[i] = the stats after step
 * first_step + i, for count consecutive steps (step 0 = the initial state),
 * each as somier_stats would have returned it right after that step. The
 * handle keeps the last SOMIER_STATS_HISTORY steps since its last
 * somier_init / somier_load (a device-side ring the step kernels write; every
 * kernel, K1_TB2's two-step launches included, computes every step's stats).
 * Errors: EINVAL (NULL with count > 0, count < 0, a step outside
 * [max(last init/load step, step_count - SOMIER_STATS_HISTORY + 1), step_count]).
 */
#define SOMIER_STATS_HISTORY 126
spread_status somier_stats_history(somier_t h, int64_t first_step, int64_t count, somier_stats_t* out);

/* Exact, order-independent combination of n partial stats (sums added as int128,
 * max of vmax2 bits); recomputes centre = sum * 2^-60 / N_total and vmax. */
spread_status somier_stats_combine(const somier_stats_t* parts, int n, const somier_params* p,
                                   somier_stats_t* out);

/*
 * somier_read -- exit-data semantics A[start:size]: copy the
 * owned planes of every chunk of this handle (and the fixed planes 0 / n0-1 held
 * as halos by the first / last chunk) into caller-owned host grids of n0*n1*n2
 * doubles each, index (i*n1 + j)*n2 + k, three separate grids per variable
 * (PAPER.md:342). Planes owned by other processes are left untouched. Blocking.
 * Any of the six pointers may be NULL to skip that grid.
 */
spread_status somier_read(somier_t h, double* x, double* y, double* z, double* vx, double* vy, double* vz);

/*
 * somier_read_planes -- `target update spread from(X[i0:count], V[i0:count])`
 * (PAPER.md:222-243): like somier_read restricted to global planes
 * [i0, i0+count); the six host grids hold count*n1*n2 doubles each (host plane
 * = global plane - i0). Planes this handle does not own are left untouched.
 * Errors: EINVAL if the range leaves [0, n0).
 */
spread_status somier_read_planes(somier_t h, int64_t i0, int64_t count, double* x, double* y, double* z, double* vx,
                                 double* vy, double* vz);

/*
 * somier_load -- update-to semantics: every owned chunk copies X[start-1 : size+2]
 * (with halos) and V[start : size] from caller-owned host grids (layout as in
 * somier_read) into device memory, and the step counter continues. Enqueued on
 * the handle's streams (asynchronous w.r.t. the host if the host memory is
 * pinned). All six pointers are required.
 */
spread_status somier_load(somier_t h, const double* x, const double* y, const double* z, const double* vx,
                          const double* vy, const double* vz);

/* Use `stream` (a cudaStream_t of the device at list position device_pos) for all
 * work of that device. NULL restores the library's own stream. */
spread_status somier_set_stream(somier_t h, int device_pos, void* stream);
spread_status somier_get_stream(somier_t h, int device_pos, void** stream);

/* Number of completed + enqueued steps. */
spread_status somier_step_count(somier_t h, int64_t* steps);

/* Number of chunks this handle owns, and K1 launches enqueued so far. */
spread_status somier_local_chunks(somier_t h, int64_t* nchunks);
spread_status somier_launch_count(somier_t h, int64_t* launches);

/* The K1 implementation this handle runs (a somier_kernel value; never
 * SOMIER_K1_AUTO): AUTO and TB2 resolve at somier_init. A K1_TB2 handle runs a
 * leftover single step (odd step count) with the same kernel in one-step mode.
 * EINVAL on NULL arguments. */
spread_status somier_kernel_in_use(somier_t h, int32_t* kernel);

/*
 * Launch timing (diagnostics; SURVEY.md §8(d) "halo time"): while on, every K1
 * launch of this handle is bracketed by three CUDA events on its stream --
 * before the neighbour-flag waits (cuStreamWaitValue64), after them (= kernel
 * start), after the kernel -- and CUDA-graph replay is off (launches are
 * enqueued one by one, without programmatic dependent launch).
 * somier_take_timing blocks, sums the recorded launches and forgets them:
 *   wait_ms    time the launches' streams sat in the flag waits, i.e. waiting
 *              for the neighbours' previous launch (their halo stores into this
 *              chunk and their skew)
 *   kernel_ms  time inside the kernels (the halo exchange is fused: the peer
 *              stores run inside the kernel)
 */
typedef struct {
    int64_t launches;
    double wait_ms, kernel_ms;          /* sums over the launches */
    double wait_max_ms, kernel_max_ms;  /* largest single launch  */
} somier_timing_t;
spread_status somier_set_timing(somier_t h, int on);
spread_status somier_take_timing(somier_t h, somier_timing_t* out);

/* Device bytes this handle allocated (all devices). */
spread_status somier_device_bytes(somier_t h, int64_t* bytes);

spread_status somier_destroy(somier_t h);

/* Library version string. */
const char* somier_version(void);

/* ------------------------------------------------------------------------
 * Host-streamed ("out-of-core") mode -- the paper's own experiment (PAPER.md
 * §V-A/B/C, 336-659): the state lives in HOST memory and
 * every time step streams it through the devices chunk by chunk:
 *   target enter data spread map(to: X[start-1:size+2], V[start:size])   (H2D)
 *   target spread ... forces/accelerations/velocities/positions/centers   (K1)
 *   target exit data spread map(from: X[start:size], V[start:size])      (D2H)
 * `buffers` device buffers per GPU: 1 = the paper's One Buffer (transfers and
 * kernels serialised per chunk); >= 2 = double buffering:
 * the H2D of the next chunk, the kernel of this one and the D2H of the
 * previous one run concurrently on three streams. Halos come from the host
 * copy of X_t (overlapping array sections), so no device-to-device
 * exchange exists in this mode.
 * ------------------------------------------------------------------------ */
typedef struct somier_stream_s* somier_stream_t;

/*
 * somier_stream_create -- s: spread over range(1 : n0-2); each chunk is the
 * slice one device processes at a time (Listing 10: chunk = buffer / ndevices).
 * buffers >= 1 device slots per list device. Device memory = buffers x
 * (3 slabs of chunk+2 planes), independent of n0: the grid may exceed HBM.
 * Errors: EINVAL, ENODEV, ENOMEM, ECUDA.
 */
spread_status somier_stream_create(spread_t s, const somier_params* p, int buffers, somier_stream_t* out);

/* As somier_stream_create with list position q on CUDA device cuda_devices[q]
 * (logical device ids, see somier_init_on); NULL = the spread's ids. */
spread_status somier_stream_create_on(spread_t s, const somier_params* p, int buffers, const int* cuda_devices,
                                      somier_stream_t* out);

/*
 * somier_stream_generate -- write the initial state (reading S7, bit-identical
 * to somier_init's) into caller-owned host grids (layout as in somier_read),
 * generated on the devices chunk by chunk. Blocking.
 */
spread_status somier_stream_generate(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                     double* vz);

/*
 * somier_stream_step -- one time step on host-resident state: reads X_t from
 * (x, y, z), writes X_{t+1} to (xn, yn, zn) -- every node, fixed faces
 * included -- and updates V = (vx, vy, vz) in place. X_t and X_{t+1} must not
 * overlap (Jacobi). `stats` (may be NULL) receives the centres / vmax of
 * X_{t+1}, V_{t+1}. Blocking. Host grids should be page-locked for the copies
 * to overlap with the kernels.
 */
spread_status somier_stream_step(somier_stream_t h, const double* x, const double* y, const double* z, double* vx,
                                 double* vy, double* vz, double* xn, double* yn, double* zn, somier_stats_t* stats);

/*
 * somier_stream_run -- nsteps time steps on host-resident state with
 * chunk-level dependencies instead of a barrier per step: the paper's future
 * work `depend(out/in: B[omp_spread_start:omp_spread_size])` on the spread
 * data directives, "making the enclosing taskgroup directive no longer
 * necessary" (Listing 13). The H2D of chunk c for step t+1
 * waits only for the D2H of chunks c-1, c, c+1 of step t, and the D2H of
 * chunk c (which overwrites X_{t-1}[c]) only for the H2D of chunks c-1, c+1 of
 * step t-1; no device idles at a step boundary. One host barrier at the end.
 *   (x, y, z) / (xn, yn, zn): the two X buffers, used alternately: step t
 *   reads the first if t is even, the second if t is odd, and writes the other
 *   one; after the call X_{nsteps} is in (x, y, z) if nsteps is even, else in
 *   (xn, yn, zn). V is updated in place. The buffers must not overlap.
 *   stats: NULL, or an array of nsteps entries receiving the statistics after
 *   each step.
 * Results are bit-identical to nsteps calls of somier_stream_step.
 * Errors: EINVAL (NULL, nsteps < 0, aliasing X buffers), ENOMEM, ECUDA.
 */
spread_status somier_stream_run(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                double* vz, double* xn, double* yn, double* zn, int64_t nsteps,
                                somier_stats_t* stats);

/*
 * somier_stream_run2 -- as somier_stream_run, but each round trip advances the
 * state TWO steps (2.5-D temporal blocking across the host link, K1_TB2):
 * per chunk map(to: X[start-2 : size+4], V[start-1 : size+2]) (clipped to the
 * grid), two fused steps, map(from: X[start : size], V[start : size]) -- half
 * the host<->device bytes per node-update of somier_stream_run. Because a
 * chunk reads its neighbours' V_t halo planes, V is double-buffered too:
 *   (x, y, z, vx, vy, vz) / (xn, ..., vzn): the two states, used alternately
 *   per launch; launch k reads the first if k is even and writes the other.
 *   nsteps / 2 two-step launches run, plus one one-step launch if nsteps is
 *   odd; the final state is in the first buffers if the number of launches
 *   is even, else in the second.
 *   stats: NULL, or an array of nsteps entries receiving the statistics after
 *   each step (both steps of a two-step launch).
 * Chunk-level dependencies as in somier_stream_run, over the chunks within
 * two planes. Results are bit-identical to somier_stream_run / the oracle.
 * Same as somier_stream_run_blocked with steps_per_trip = 2 (its device
 * buffers are allocated on first use).
 * Errors: EINVAL (NULL, nsteps < 0, aliasing buffers), ENOMEM, ECUDA.
 */
spread_status somier_stream_run2(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                 double* vz, double* xn, double* yn, double* zn, double* vxn, double* vyn,
                                 double* vzn, int64_t nsteps, somier_stats_t* stats);

/*
 * somier_stream_run_blocked -- as somier_stream_run2 with `steps_per_trip` = s
 * steps per host round trip (1 <= s <= 256; s = 2 is somier_stream_run2): per
 * chunk map(to: X[start-s : size+2s], V[start-v : size+2v]) with v =
 * max(1, s-1) (clipped to the grid), ceil(s/2) K1_TB2 launches over
 * regions that shrink by two planes per side per launch down to the chunk
 * itself (an odd s ends with a one-step launch), map(from: X[start : size],
 * V[start : size]). Host<->device bytes per node-update fall as ~1/s while
 * the device recomputes the overlap (a chunk of S planes computes ~S + s
 * planes per step on average). Buffers alternate per trip as in run2 (the
 * final state is in the first buffers if the number of trips ceil(nsteps/s)
 * is even); stats: NULL or nsteps entries, one per step (every launch of a
 * trip counts the chunk's own planes only).
 * Device memory: `buffers` x 2 x (X and V of max_chunk + 2s + 2 planes) per
 * device, allocated on first use. Bit-identical to somier_stream_run.
 * Errors: EINVAL, ENOMEM, ECUDA.
 */
spread_status somier_stream_run_blocked(somier_stream_t h, double* x, double* y, double* z, double* vx, double* vy,
                                        double* vz, double* xn, double* yn, double* zn, double* vxn, double* vyn,
                                        double* vzn, int64_t nsteps, int64_t steps_per_trip, somier_stats_t* stats);

/* Bytes moved host->device and device->host by one trip of
 * somier_stream_run_blocked with s steps. */
spread_status somier_stream_traffic_blocked(somier_stream_t h, int64_t steps_per_trip, int64_t* h2d_bytes,
                                            int64_t* d2h_bytes);

/* Bytes moved host->device and device->host by one somier_stream_step (one
 * step of somier_stream_run), and K1 launches so far. */
spread_status somier_stream_traffic(somier_stream_t h, int64_t* h2d_bytes, int64_t* d2h_bytes, int64_t* launches);

/* Bytes moved host->device and device->host by one two-step launch of
 * somier_stream_run2. */
spread_status somier_stream_traffic2(somier_stream_t h, int64_t* h2d_bytes, int64_t* d2h_bytes);

/* Chunk tasks (one chunk mapped in, stepped, mapped out) each list position has
 * run since the handle was created; counts[] holds one entry per position. With
 * spread_schedule(dynamic) these show how the chunks were shared out. */
spread_status somier_stream_chunk_counts(somier_stream_t h, int64_t* counts);

/* Test hook: every chunk task of list position device_pos first spins >= ns
 * nanoseconds on that device (a deliberately slower device, to exercise the
 * dynamic schedule); 0 switches it off. */
spread_status somier_stream_set_delay(somier_stream_t h, int device_pos, int64_t ns);

spread_status somier_stream_destroy(somier_stream_t h);

#ifdef __cplusplus
}
#endif
#endif /* PAPER_SOMIER_H */
