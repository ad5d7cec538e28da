/*
 * tg.h -- C ABI of the B200-native out-of-core operator-graph executor.
 *
 * Method: N. Sundaram, A. Raghunathan, S. T. Chakradhar, "A framework for efficient and
 * scalable execution of domain-specific templates on GPUs", IPDPS 2009. The
 * user-facing contract of the paper is: templates are parametrized APIs (PAPER.md:51,
 * :623 `edge_map = find_edges(Image, Kernel, num_orientations, Combine_op)`); a template
 * is a graph of parallel operators with statically known footprints and splitting rules
 * (PAPER.md:345, :349 fn. 1); the target GPU is described by parameters such as its
 * memory capacity (Fig. 4, "Total GPU Memory" PAPER.md:409); the framework
 * derives an execution plan and a run-time library executes it.
 *
 * Conventions for every function below:
 *  - Return value: tg_status, TG_OK (0) on success, a negative TG_E_* code on failure.
 *    No C++ exception or longjmp crosses this ABI. On failure tg_last_error() returns a
 *    thread-local, NUL-terminated message describing the last failure of that thread.
 *  - Data structures (DS) are dense fp32 arrays in [n][c][h][w] order (row-major, w
 *    fastest), the paper's "floats". A DS is identified by a tg_id >= 0.
 *  - Host buffers passed in are CALLER-OWNED; they must stay valid and unchanged (inputs,
 *    parameters) or untouched (outputs) until tg_execute returns (or, for
 *    tg_execute_async, until the compute stream reaches the end of the execution).
 *    Pinned (page-locked) host memory is used as is; pageable memory of 1 MiB or more is
 *    registered with cudaHostRegister at the first execution (a failure is TG_E_CUDA, never a
 *    silent fall-back to pageable copies) and unregistered by tg_plan_destroy.
 *  - Device memory is owned by the library: per device it obtains exactly ONE arena of
 *    tg_plan_stats.peak_device_bytes bytes (never more than the device budget) through
 *    tg_runtime.alloc (or cudaMalloc when no runtime is set) and returns it at
 *    tg_plan_destroy. Device-resident inputs/outputs (tg_input_device/tg_output_device)
 *    are caller-owned device buffers on the plan's device (one-device plans only). Their
 *    producer and consumer are ordered against the execution through a caller stream:
 *    tg_execute_on's `stream`, or for tg_execute / tg_execute_async the legacy default
 *    stream (cudaStreamLegacy, where PyTorch's default stream enqueues).
 *  - Threading: a graph is not thread-safe while it is being built; a plan may be
 *    executed repeatedly but by one thread at a time; independent plans may run
 *    concurrently on disjoint devices.
 */
#ifndef TG_H
#define TG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t tg_status;
#define TG_OK 0
#define TG_E_ARG (-1)          /* bad argument (NULL pointer, unknown id, bad enum)      */
#define TG_E_SHAPE (-2)        /* shapes of the operands do not agree                    */
#define TG_E_INFEASIBLE (-3)   /* the budget cannot hold even the smallest chunk of a unit
                                  (unsplittable operators must fit)        */
#define TG_E_CUDA (-4)         /* a CUDA runtime call failed (message has the CUDA error)*/
#define TG_E_OOM (-5)          /* host or device allocation failed                       */
#define TG_E_STATE (-6)        /* call not valid in the current state                    */
#define TG_E_UNSUPPORTED (-7)  /* graph/mode combination not implemented                 */

typedef struct tg_graph tg_graph;
typedef struct tg_plan tg_plan;
typedef int32_t tg_id;

/* enums */
#define TG_VALID 0        /* conv2d: output (H-k+1) x (W-k+1)                            */
#define TG_SAME 1         /* conv2d: output H x W, zero padding (k-1)/2 top/left, k/2
                             bottom/right (reading R2)                         */
#define TG_ADD 0          /* elementwise y = x0 + x1 + ... (left to right)                */
#define TG_NEG 1          /* elementwise y = -x0  (the edge template's "remap" R, R3)     */
#define TG_AFFINE 2       /* elementwise y = a * x0 + b                                   */
#define TG_ABS 3          /* elementwise y = |x0|                                         */
#define TG_MAX 0          /* combine op of tg_find_edges                                  */
#define TG_SUM 1          /* combine op: sum of the convolutions' responses              */
#define TG_MAXABS 2       /* combine op: max of |response|                                */
#define TG_BIAS_PLANE 0   /* CNN bias: one full plane per output map (the paper's Fig. 7)
                             shape [1][c][h][w], shared by every image of the batch       */
#define TG_BIAS_SCALAR 1  /* CNN bias: one scalar per output map, shape [c]               */
#define TG_FP32 0         /* all arithmetic in fp32 (FFMA); parity 1e-5 normwise          */
#define TG_BF16_TC 1      /* CNN C3/C5/C6 on tcgen05 tensor cores, bf16 operands, fp32
                             accumulation; parity 2e-2 normwise                           */
#define TG_FP32_TC 2      /* fp32-accurate CNN with C3 and C5 on tcgen05: every operand scaled
                             by a power of two and split into two fp16 numbers, three MMAs
                             per product (3xFP16), fp32 accumulation; parity 1e-5 normwise
                             like TG_FP32                                                   */
#define TG_FUSED 0        /* offload units = fused templates (edge: 1 unit; CNN: 3)       */
#define TG_PER_OP 1       /* paper mode: operators that exceed the budget are split into row
                             pieces (R19), one operator piece
                             per offload unit, DFS order + latest-time-of-use
                             transfers, one stream, generic kernels    */
#define TG_BASELINE 2     /* paper baseline: per operator copy inputs in,
                             run, copy outputs out, keep nothing                          */

/* ------------------------------------------------------------------ graph building */
tg_status tg_graph_create(tg_graph** g);
void tg_graph_destroy(tg_graph* g);

/* Template input (image batch) in HOST memory: [n][c][h][w] fp32, caller-owned. */
tg_status tg_input(tg_graph* g, int64_t n, int64_t c, int64_t h, int64_t w, const float* host,
                   tg_id* out);
/* Template input already resident in DEVICE memory of the plan's device (in-core runs). */
tg_status tg_input_device(tg_graph* g, int64_t n, int64_t c, int64_t h, int64_t w,
                          const float* dev, tg_id* out);
/* Parameter (kernel, bias, subsample weights) in HOST memory, shape [d0][d1][d2][d3]
 * (unused leading dims = 1). Parameters are never split. */
tg_status tg_param(tg_graph* g, int64_t d0, int64_t d1, int64_t d2, int64_t d3,
                   const float* host, tg_id* out);
/* 2-D cross-correlation (reading R1) of every input plane with k[co][ci][kh][kw], summed
 * over ci (a fully connected conv layer; Fig. 7 PAPER.md:641-713 is its per-pair
 * expansion), plus an optional bias (-1 = none; [co] scalars or a plane [1][co][ho][wo]
 * shared over n). pad = TG_VALID | TG_SAME. */
tg_status tg_conv2d(tg_graph* g, tg_id x, tg_id k, tg_id bias, int32_t pad, tg_id* y);
/* Elementwise op over same-shaped DS (op = TG_ADD | TG_NEG | TG_AFFINE | TG_ABS). */
tg_status tg_elementwise(tg_graph* g, int32_t op, const tg_id* xs, int32_t nx, float a,
                         float b, tg_id* y);
tg_status tg_tanh(tg_graph* g, tg_id x, tg_id* y);
/* n-ary max: y = left fold (x_k > m) ? x_k : m over xs in order (reading R5). */
tg_status tg_max_combine(tg_graph* g, const tg_id* xs, int32_t nx, tg_id* y);
/* Subsample: window s, stride s, kernel p[c][s][s] per plane (reading R8). */
tg_status tg_subsample(tg_graph* g, tg_id x, tg_id p, int32_t s, tg_id* y);
/* Bind template output y to caller-owned HOST memory sized by tg_shape(y). */
tg_status tg_output(tg_graph* g, tg_id y, float* host_dst);
/* Bind template output y to caller-owned DEVICE memory on the plan's device. */
tg_status tg_output_device(tg_graph* g, tg_id y, float* dev_dst);
/* dims = {n, c, h, w} of DS id. */
tg_status tg_shape(const tg_graph* g, tg_id id, int64_t dims[4]);

/* Template helpers (PAPER.md:623 find_edges; PAPER.md:635 the CNN built from torch5
 * primitives). Both only append primitive nodes to the graph. */
/* Edge detection: num_orientations (2, 4 or 8) orientations in steps of
 * 360/num_orientations degrees; the first half are SAME convolutions of img with `kernel`
 * ([1][1][k][k], k <= 16) rotated on the host (multiples of 90 degrees exactly, others by
 * bilinear interpolation, R18), the second half their remaps (negations).
 * combine_op: TG_MAX (max over all orientations), TG_MAXABS (max |response| of the
 * convolutions), TG_SUM (sum of the convolutions; the remaps would cancel). TG_FUSED runs
 * any of these as one kernel (up to 4 convolutions). */
tg_status tg_find_edges(tg_graph* g, tg_id img, tg_id kernel, int32_t num_orientations,
                        int32_t combine_op, tg_id* edge_map);
/* CNN of SURVEY F2 (11 layers): C1(1->8,5x5) T S2 T C3(8->20,5x5) T S4 T C5(20->n5,5x5)
 * T C6(n5->9,1x1); 1 <= n5 <= 128 (small net 20, large net 120). params order: K1[8][1][5][5],
 * B1, P2[8][2][2], K3[20][8][5][5], B3, P4[20][2][2], K5[n5][20][5][5], B5, K6[9][n5][1][1],
 * B6; Bk = plane [1][c][h][w] (TG_BIAS_PLANE) or [c] (TG_BIAS_SCALAR). */
tg_status tg_cnn(tg_graph* g, tg_id img, int32_t n5, const tg_id params[10], int32_t bias_mode,
                 tg_id* out);

/* Matrix-matrix multiply C = A B: a [1][1][m][k], b [1][1][k][n] (any DS
 * kinds), result [1][1][m][n]. When it does not fit, TG_PER_OP splits it by rows of A and C,
 * B read whole ("breaking up one of the input matrices and the output matrix", DESIGN.md
 * R20). fp32 with fp32 accumulation in order l = 0..k-1. TG_E_SHAPE if the inner dimensions
 * differ or an operand is not a matrix. Executed by TG_PER_OP / TG_BASELINE plans (TG_FUSED
 * plans only the edge and CNN templates: TG_E_UNSUPPORTED). */
tg_status tg_matmul(tg_graph* g, tg_id a, tg_id b, tg_id* y);

/* ------------------------------------------------------------------ target parameters */
/* Devices the plan runs on (one host thread per device; chunks are split contiguously).
 * Default: the current CUDA device. Plans with device-resident I/O take one device
 * (TG_E_UNSUPPORTED at tg_plan_create otherwise). */
tg_status tg_set_devices(tg_graph* g, const int32_t* ordinals, int32_t n);
/* Device-memory budget per device in bytes ("Total GPU Memory"); 0 =
 * uncapped. The plan's arena never exceeds it. */
tg_status tg_set_device_budget(tg_graph* g, uint64_t bytes_per_device);
tg_status tg_set_precision(tg_graph* g, int32_t prec);
/* Input pixels per chunk when memory does not bind (default 1<<25) and pipeline depth
 * (in-flight chunk slots, default 3, 1..8). */
tg_status tg_set_chunking(tg_graph* g, int64_t max_chunk_px, int32_t depth);
/* Multi-process sharding: this process executes chunk range [floor(C*rank/world),
 * floor(C*(rank+1)/world)) of the global chunk list (no collective). The chunk
 * list is the same for every world size, so outputs are bit-identical across world sizes.
 * The template input and output buffers are only read and written over the span of this
 * shard's chunks (tg_plan_stats chunk_begin/chunk_end; the JSON plan lists each chunk's rows):
 * a process may pass a base pointer whose other parts are not mapped, holding only its share
 * of a global host input (only that span is page-locked). */
tg_status tg_set_shard(tg_graph* g, int32_t rank, int32_t world);

/* Runtime hooks (PyTorch-backed in the Python binding). alloc returns device memory on
 * `dev` (NULL on failure); stream returns a cudaStream_t for which = 0 (H2D), 1 (compute),
 * 2 (D2H). Any member may be NULL (library default). The struct is copied. */
typedef struct {
    void* (*alloc)(size_t bytes, int32_t dev, void* ctx);
    void (*free)(void* ptr, int32_t dev, void* ctx);
    void* (*stream)(int32_t dev, int32_t which, void* ctx);
    void* ctx;
} tg_runtime;
tg_status tg_set_runtime(tg_graph* g, const tg_runtime* rt);

/* ------------------------------------------------------------------ plan / execute */
/* Build the execution plan: recognise the template's offload units, split into chunks
 * (PAPER.md:359-371), order them and size every transfer. Pure host
 * code: works without a GPU. mode = TG_FUSED (edge/CNN templates, split into chunks);
 * TG_PER_OP (any graph, host I/O, one device: operators that do not fit within 7/8 of the
 * budget are split into row pieces, PAPER.md:359-367 / DESIGN.md R19 -- TG_E_INFEASIBLE if
 * even single-row pieces do not fit, TG_E_UNSUPPORTED if a whole-read operand would span
 * more than 8 pieces); TG_BASELINE (any graph, operators run whole: TG_E_INFEASIBLE if one
 * does not fit). The graph must outlive the plan. */
tg_status tg_plan_create(const tg_graph* g, int32_t mode, tg_plan** plan);

typedef struct {
    uint64_t h2d_bytes;              /* predicted host->device bytes of this shard      */
    uint64_t d2h_bytes;              /* predicted device->host bytes of this shard      */
    uint64_t io_lower_bound_bytes;   /* template inputs + params + outputs, once        */
    uint64_t total_temp_bytes;       /* sum of all DS at Fig. 7 granularity (Table 1)   */
    uint64_t peak_device_bytes[8];   /* arena bytes per device of the plan              */
    int64_t n_chunks;                /* global chunk count                              */
    int64_t n_units;                 /* fused offload units per chunk                   */
    int64_t n_ops_fig7;              /* operators of the template at Fig. 7 granularity */
    int64_t n_ds_fig7;               /* data structures at Fig. 7 granularity           */
    int64_t chunk_begin, chunk_end;  /* this shard's chunk range                        */
    uint64_t host_registered_bytes;  /* pageable host bytes registered by the library   */
    uint64_t h2d_bytes_steady;       /* H2D bytes of a later execution: parameters stay
                                        resident in the arena after the first one        */
    uint64_t io_lower_bound_data_bytes; /* io_lower_bound_bytes without the parameters: the
                                        floor of h2d_bytes_steady + d2h_bytes (images in,
                                        outputs out, once)                               */
} tg_plan_stats;
tg_status tg_plan_stats_get(const tg_plan* plan, tg_plan_stats* out);

/* Plan as JSON (chunks with halo row ranges, slot layout, byte counts); compared
 * bit-exactly with the planner oracle. Writes at most cap bytes incl. NUL; *needed =
 * required size incl. NUL. Returns TG_E_ARG when buf is too small (buf may be NULL). */
tg_status tg_plan_dump_json(const tg_plan* plan, char* buf, size_t cap, size_t* needed);

/* Execute the plan; blocks until outputs are valid in their destinations. */
tg_status tg_execute(tg_plan* plan);
/* Same, but returns once all work is enqueued; completion is ordered before any later work
 * on the compute stream (which = 1) of every device of the plan. Back-to-back executions
 * of one host-I/O plan pipeline: the next execution's first H2D copies may run while the
 * previous one's last chunks compute and download (each copy waits only for its slot). */
tg_status tg_execute_async(tg_plan* plan);

/* Same as tg_execute (blocking != 0) or tg_execute_async, ordered against a caller stream
 * (a cudaStream_t of the plan's device; NULL = the legacy default stream): the execution starts
 * after all work enqueued on `stream` before the call, and work enqueued on `stream` after the
 * call starts after the execution completes. Fused plans on one device; TG_E_UNSUPPORTED
 * otherwise. */
tg_status tg_execute_on(tg_plan* plan, void* stream, int32_t blocking);

/* CUDA-graph replay (fused plans, one device): with on != 0 the next execution after the
 * parameters are resident is captured (its copies, kernels and stream dependencies on the
 * three streams) and that and every later execution launch the captured graph on the compute
 * stream -- one host call instead of one per copy and kernel, which is what bounds small
 * (launch-latency-bound) executions. Replays are serialised on the compute stream, so
 * back-to-back executions no longer overlap each other's copies. Ignored while profiling;
 * tg_plan_invalidate_params or on = 0 drops the graph. Buffers must not move between
 * executions (they never do: the plan binds them). */
tg_status tg_plan_set_graph(tg_plan* plan, int32_t on);

/* Per-launch timing of the fused kernels measured with CUDA events on the compute stream
 * (enable before executing; tg_plan_timing_get synchronizes). Times are summed over all
 * executions since enabling. on = 1: kernels and every H2D/D2H copy (events on the copy
 * streams make a copy engine finish one copy before starting the next, so streamed steps
 * slow down); on = 2: kernels only (no events on the copy streams); 0: off. */
typedef struct {
    int64_t launches;        /* kernel launches of the library                          */
    int64_t executions;
    double kernel_ms[4];     /* per unit kind: 0 edge, 1 CNN U1, 2 CNN U2, 3 CNN U3     */
    int64_t unit_launches[4];
    double h2d_ms, d2h_ms;   /* summed copy durations (copy streams)                    */
} tg_timing;
tg_status tg_plan_set_profiling(tg_plan* plan, int32_t on);
tg_status tg_plan_timing_get(tg_plan* plan, tg_timing* out);

/* Timeline of the profiled copies and launches (fused mode): one record per H2D chunk copy,
 * kernel launch and D2H chunk copy, in enqueue order, with start/end in ms relative to the
 * first profiled record of its device in the batch collected. Collected (and appended) by
 * tg_plan_timing_get / this call, which synchronize; cleared by tg_plan_set_profiling(1).
 * Writes min(cap, total) records to out (out may be NULL when cap == 0); *n = total. */
typedef struct {
    int32_t device;
    int32_t kind;            /* 0 edge, 1..3 CNN U1..U3, 10 H2D copy, 11 D2H copy        */
    int64_t chunk;           /* chunk index within the plan (-1: parameter upload)       */
    double t0_ms, t1_ms;
} tg_trace_rec;
tg_status tg_plan_trace_get(tg_plan* plan, tg_trace_rec* out, size_t cap, size_t* n);
/* Parameters are copied to the device by the first execution of a plan and stay resident
 * in its arena; call this after changing parameter host data to re-upload them at the next
 * execution. */
tg_status tg_plan_invalidate_params(tg_plan* plan);
/* Kernel launches issued by the library since plan creation (always counted). */
int64_t tg_plan_launch_count(const tg_plan* plan);

void tg_plan_destroy(tg_plan* plan);

/* ------------------------------------------------------------------ operator library */
/* The operator library of Fig. 4: one call runs output rows [r0, r1) of one
 * operator -- a piece of a split operator or the whole operator -- on the
 * device. TG_PER_OP / TG_BASELINE plans execute through it, and the code generator below emits
 * calls to it. All pointers are DEVICE pointers owned by the caller. A data structure piece
 * holding rows [r0, r1) of a DS [n][c][h][w] is stored [n][c][r1-r0][w]; an input is a view
 * of up to TG_OPLIB_MAX_SEG such pieces (a row is read from the first piece that holds it;
 * overlapping pieces must hold identical rows). Returns TG_E_ARG for malformed descriptors
 * (unknown kind, too many inputs/pieces, a kernel or subsample weight not in one piece at row
 * 0), TG_E_CUDA if the launch fails; the call is asynchronous on `stream` (a cudaStream_t,
 * NULL = legacy default stream). */
#define TG_OPLIB_MAX_SEG 8
#define TG_OPLIB_MAX_IN 16
#define TG_OPLIB_CONV 0     /* in: x, kernel[, bias] ; pad, dims as tg_conv2d              */
#define TG_OPLIB_ELEM 1     /* in: xs ; elem = TG_ADD..TG_ABS, 4 = tanh, 5 = max; a, b       */
#define TG_OPLIB_SUB 2      /* in: x, p ; s                                                 */
#define TG_OPLIB_MATMUL 3   /* in: a, b (b read whole)                                      */
typedef struct {
    const float* p;         /* piece buffer [n][c][r1-r0][w]                                */
    int64_t r0, r1;         /* rows of the DS it holds                                      */
} tg_oplib_seg;
typedef struct {
    tg_oplib_seg seg[TG_OPLIB_MAX_SEG];
    int32_t nseg;
} tg_oplib_view;
typedef struct {
    int32_t kind;                       /* TG_OPLIB_*                                        */
    int32_t nin;                        /* inputs used in in[] / in_dims[]                   */
    tg_oplib_view in[TG_OPLIB_MAX_IN];
    int64_t in_dims[TG_OPLIB_MAX_IN][4];  /* [n][c][h][w] of each input DS                   */
    float* y;                           /* output piece: rows [r0, r1) of y_dims, [n][c][r1-r0][w] */
    int64_t y_dims[4];
    int64_t r0, r1;
    int32_t pad;                        /* conv: TG_VALID | TG_SAME                          */
    int32_t elem;                       /* elementwise op (see TG_OPLIB_ELEM)                */
    int32_t s;                          /* subsample window = stride                         */
    float a, b;                         /* TG_AFFINE coefficients                            */
} tg_oplib_op;
tg_status tg_oplib_run(const tg_oplib_op* op, void* stream);

/* Code generator ("A code generator takes the execution plan generated by the
 * previous steps, and generates a hybrid CPU/GPU program ... compiled together with a larger
 * application"): C source replaying a TG_PER_OP / TG_BASELINE plan -- every H2D copy of a
 * piece (2-D copies of its rows), every tg_oplib_run call, every D2H copy, with the plan's
 * static arena offsets baked in. The source defines
 *   int tg_generated_execute(float* const* host, char* arena, void* stream);
 *   TG_GEN_ARENA_BYTES, TG_GEN_NUM_DS
 * where host[d] is the host buffer of graph DS d (inputs, parameters and the output; others
 * may be NULL), arena a device buffer of TG_GEN_ARENA_BYTES bytes, stream a cudaStream_t; it
 * returns 0 when the output is complete on the host, a tg_status otherwise. Compile with the
 * CUDA runtime headers and link against this library and cudart. Writes at most cap bytes
 * incl. NUL; *needed = required size incl. NUL; TG_E_ARG if buf is too small,
 * TG_E_UNSUPPORTED for TG_FUSED plans. */
tg_status tg_plan_codegen(const tg_plan* plan, char* buf, size_t cap, size_t* needed);

/* ------------------------------------------------------------------ transfer scheduling */
/* The paper's heuristic offload/transfer scheduler (Section 3.3.1) over an
 * abstract operator graph whose data structures have sizes in any unit (floats, bytes, or
 * the "units" of Fig. 3). Pure host code. */
typedef struct tg_sched tg_sched;
#define TG_DS_INPUT 0   /* template input: starts valid on the host                      */
#define TG_DS_PARAM 1   /* parameter: starts valid on the host                           */
#define TG_DS_TEMP 2    /* intermediate: produced by an operator                         */
#define TG_DS_OUTPUT 3  /* template output: must end on the host (PB constraint (13))    */
tg_status tg_sched_create(tg_sched** s);
void tg_sched_destroy(tg_sched* s);
tg_status tg_sched_add_ds(tg_sched* s, uint64_t size, int32_t kind, int32_t* id);
/* An operator reading ins[0..nin) and writing outs[0..nout) (DS ids). */
tg_status tg_sched_add_op(tg_sched* s, const int32_t* ins, int32_t nin, const int32_t* outs, int32_t nout,
                          int32_t* id);
/* Depth-first operator schedule: order[0..n_ops) receives operator ids.
 * Children are consumers in insertion order, start nodes in id order (R11). */
tg_status tg_sched_dfs_order(const tg_sched* s, int32_t* order);
/* "Latest time of use" transfer schedule for a given operator order (read
 * as next use, R10) within `capacity`: *moved = total size copied host<->GPU.
 * If trace != NULL it receives (kind, id) pairs -- kind 0 = copy DS id to the GPU, 1 = run
 * operator id, 2 = copy DS id to the host; trace_cap counts pairs; *trace_len = pairs used.
 * TG_E_INFEASIBLE if an operator's inputs and outputs do not fit together. */
tg_status tg_sched_transfers(const tg_sched* s, const int32_t* order, uint64_t capacity, uint64_t* moved,
                             int32_t* trace, int64_t trace_cap, int64_t* trace_len);
/* Exact counterpart of the heuristic for small graphs: the minimum of the
 * transfer volume of tg_sched_transfers over EVERY operator order that respects the data
 * dependences (PB constraints (1)-(3) of Fig. 5; the paper solved the full
 * PB model with MiniSAT+, PAPER.md:477 -- here the eviction policy stays next-use, DESIGN.md
 * R10, and the search is over operator orders). order[0..n_ops) receives the lexicographically
 * smallest optimal order, *moved its volume, *n_orders (may be NULL) the number of orders
 * enumerated and *n_optimal (may be NULL) how many reach the minimum.
 * TG_E_UNSUPPORTED if the graph has more than max_orders orders (the enumeration is
 * factorial: meant for graphs of ~12 operators or fewer); TG_E_INFEASIBLE if no order fits. */
tg_status tg_sched_optimal(const tg_sched* s, uint64_t capacity, uint64_t max_orders, int32_t* order,
                           uint64_t* moved, uint64_t* n_orders, uint64_t* n_optimal);

/* ------------------------------------------------------------------ measurement */
/* Measured FP32 FFMA peak of `device` in TFLOP/s (2 flop per FMA lane): a probe kernel of
 * independent paired-FMA (FFMA2) chains over every SM, best of a few launches of tens of ms,
 * at the clocks the device runs at. The denominator of the ALU-bound rooflines (not part of
 * the paper's method). Synchronizes the device; TG_E_CUDA on failure. */
tg_status tg_probe_fp32_peak(int32_t device, double* tflops);

const char* tg_last_error(void);
/* Library version string, e.g. "tg 0.1 sm_100a". */
const char* tg_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TG_H */
