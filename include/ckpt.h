/*
 * ckpt.h -- C ABI of libckpt.so, the B200 (sm_100a) hot path of
 *   Tan et al., "Towards Affordable Reproducibility Using Scalable Capture
 *   and Comparison of Intermediate Multi-Run Results", MIDDLEWARE '24.
 *   ("P:<line>" = line of /root/reference/PAPER.md; "R<k>" = a reading in
 *   DESIGN.md section "Readings of the paper".)
 *
 * Problem: given the checkpoints of two runs, list every datum
 * (with its index) whose values differ by more than a user bound eps,
 * |V_A - V_B| > eps.  The method (Alg. 1):
 *   1. split each checkpoint array into fixed-size chunks, conservatively
 *      round every float to the bound and hash each chunk with block-chained
 *      128-bit Murmur3F into a Merkle leaf              -> ckpt_tree_build*
 *   2. build the Merkle tree level by level               -> ckpt_tree_build*
 *   3. BFS both trees top-down from a mid level, pruning equal subtrees,
 *      to list the chunks whose leaves differ            -> ckpt_tree_diff*
 *   4. compare only those chunks element by element      -> ckpt_verify*
 *
 * Conventions for every entry point
 * ---------------------------------
 *  - Pointers are CUDA DEVICE pointers of the device that is current on
 *    the calling thread, unless the parameter is marked (host).
 *  - `stream` is a cudaStream_t (NULL = legacy default stream).  All device
 *    work is enqueued on it.  Functions that return a count through a
 *    (host) pointer synchronise `stream` before returning; functions named
 *    *_async never synchronise.
 *  - Input arrays are borrowed: caller-owned, unmodified, and they must stay
 *    valid until the enqueued work completes.  Data pointers must be 16-byte
 *    aligned (the leaf kernel moves 16-byte blocks).
 *  - Trees are library-owned (opaque); release with ckpt_tree_free*.
 *  - Output buffers are caller-allocated with capacity `cap` entries.  When
 *    the full count exceeds `cap`, the first `cap` entries (ascending) are
 *    written, the full count is still returned and the status is
 *    CKPT_ETRUNC.
 *  - Outputs are unique, ascending, 0-based ids (R17).  For a checkpoint of
 *    several arrays, ids are global: array a's chunk c is
 *    chunk_base[a] + c and its element i is elem_base[a] + i, where the
 *    bases are the running sums of the arrays' chunk / element counts in
 *    array order.
 *  - Errors never abort the process.  CKPT_ECUDA carries the CUDA error
 *    text, retrievable with ckpt_last_error() (thread-local).
 *  - There is no CPU fallback: without a usable sm_100 device every
 *    compute entry point returns CKPT_ECUDA.
 */
#ifndef CKPT_H
#define CKPT_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    CKPT_OK = 0,
    CKPT_EINVAL = -1,    /* bad argument (see each function) */
    CKPT_EMISMATCH = -2, /* trees not built with the same shape / parameters (R19) */
    CKPT_ENOMEM = -3,    /* device allocation failed */
    CKPT_ECUDA = -4,     /* CUDA runtime / launch error */
    CKPT_ETRUNC = -5     /* output longer than `cap`; first `cap` entries valid */
} ckpt_status;

typedef enum { CKPT_F32 = 0, CKPT_F64 = 1 } ckpt_dtype;  /* HACC fields are F32 */

typedef struct ckpt_tree ckpt_tree;

/* ------------------------------------------------------------------------
 * Step 1+2: capture-time tree construction (Alg. 1; P:463-474;
 * section 2.4).
 *
 * Chunking (R12): chunk c of an array covers input bytes
 * [c*chunk_bytes, min(nbytes, (c+1)*chunk_bytes)); chunk_bytes must be a
 * positive multiple of 16 (one 128-bit hash block).
 * Rounding (R5-R9): inv = RN(1/eps); every element x becomes
 * k = clamp(floor(x * inv)) (exact product; NaN -> 0); the hashed word is
 * k's low 32 bits for F32 and all 64 bits for F64.  eps == 0 hashes the raw
 * element bits (R10).
 * Leaf (R2-R4): (h1,h2) = (0,0); for every 16-byte block of
 * words, (h1,h2) = MurmurHash3_x64_128(block, len, state (h1,h2)); a final
 * block shorter than 16 bytes uses Murmur3F's tail.  leaf = h1 || h2.
 * Levels (R13-R14): n_{l+1} = ceil(n_l/2); node = Murmur3F(left
 * || right, 32 bytes, seed 0) or the left child promoted when it has no
 * sibling.
 * Checkpoint of several arrays (R15): every array gets its own tree; the
 * checkpoint root is the same level construction over the array roots in
 * array order.
 *
 * Arguments:
 *   data        device pointer to n elements of `dtype`, little-endian,
 *               16-byte aligned.
 *   n           element count, >= 1.
 *   eps         absolute bound, finite and >= 0.
 *   out (host)  receives the new tree.
 * The build is asynchronous on `stream`; the tree may be used by later
 * work on the same stream (or after synchronising it).
 * Errors: CKPT_EINVAL for n == 0, NULL pointers, misaligned data,
 * chunk_bytes == 0 or not a multiple of 16, eps < 0 / NaN / inf, unknown
 * dtype; CKPT_ENOMEM; CKPT_ECUDA.
 * ---------------------------------------------------------------------- */
ckpt_status ckpt_tree_build(const void *data, uint64_t n, ckpt_dtype dtype, uint32_t chunk_bytes,
                            double eps, void *stream, ckpt_tree **out);

/* Same for a checkpoint made of n_arrays >= 1 arrays (e.g. the six HACC
 * particle fields of one rank).  data (host) and n (host) are arrays of
 * n_arrays device pointers / element counts.  All arrays are hashed in one
 * leaf-kernel launch. */
ckpt_status ckpt_tree_build_arrays(const void *const *data, const uint64_t *n, uint32_t n_arrays,
                                   ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                                   void *stream, ckpt_tree **out);

/* Several checkpoints' trees with ONE leaf-kernel launch (e.g. run A and run B
 * of a pair, so the leaf kernel's last wave of chunk chains is fuller).
 * data (host) / n (host) list the arrays of all trees back to back;
 * arrays_per_tree (host, n_trees entries) splits them; out (host, n_trees
 * entries) receives the trees.  Same rules and errors as
 * ckpt_tree_build_arrays; on error no tree is returned. */
ckpt_status ckpt_tree_build_batch(const void *const *data, const uint64_t *n,
                                  const uint32_t *arrays_per_tree, uint32_t n_trees,
                                  ckpt_dtype dtype, uint32_t chunk_bytes, double eps, void *stream,
                                  ckpt_tree **out);

/* Hash-block variant (reading R23).  The paper hashes 128-bit blocks
 * and notes that "the block size is variable and can be adjusted":
 * the chain of the leaf runs over blocks of hash_block bytes, each block one
 * complete Murmur3F call seeded with the previous digest; a chunk's last block
 * holds the bytes that remain and is hashed with its own length.
 *   hash_block  16 = the default of every other entry point; any positive
 *               multiple of 16; 0 (or >= chunk_bytes) = the whole chunk in one
 *               Murmur3F call, seed 0.
 * Larger blocks finalise less often (fewer instructions per byte); the
 * quantizer, the tree levels, diff and verify are unchanged, and the set of
 * flagged chunks is the same (barring 2^-128 collisions).  Trees of different
 * hash_block are incompatible (CKPT_EMISMATCH in diff).  Errors as
 * ckpt_tree_build_batch, plus CKPT_EINVAL when hash_block % 16 != 0. */
ckpt_status ckpt_tree_build_batch_ex(const void *const *data, const uint64_t *n,
                                     const uint32_t *arrays_per_tree, uint32_t n_trees,
                                     ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                                     uint32_t hash_block, void *stream, ckpt_tree **out);

/* Tree over caller-supplied 16-byte digests used as leaves (no data
 * hashing).  Used to form the top levels over the subtree roots gathered
 * from all GPUs (R15; the multi-GPU path).  digests16: device, count*16
 * bytes.  The result supports ckpt_tree_root / ckpt_tree_nodes only. */
ckpt_status ckpt_tree_from_digests(const void *digests16, uint64_t count, void *stream,
                                   ckpt_tree **out);

/* n_trees such trees with ONE interior-level launch (the multi-GPU step
 * builds the top trees of run A and run B together).  digests16: device,
 * the counts[k] digests of tree k follow those of tree k-1; counts: host,
 * n_trees entries, each > 0; out: host array of n_trees handles (all NULL on
 * error).  Same result as n_trees calls of ckpt_tree_from_digests. */
ckpt_status ckpt_tree_from_digests_batch(const void *digests16, const uint64_t *counts,
                                         uint32_t n_trees, void *stream, ckpt_tree **out);

/* Release a tree.  ckpt_tree_free orders the release after the work on the
 * tree's build stream (which must still exist); ckpt_tree_free_on orders it
 * on `stream` instead.  NULL is ignored. */
void ckpt_tree_free(ckpt_tree *t);
void ckpt_tree_free_on(ckpt_tree *t, void *stream);

/* ------------------------------------------------------------------------
 * Step 3: stage-1 comparison, BFS with pruning (P:555-566, P:642-648,
 * Fig. 4; R16).  Starts at the level l0 closest to the root whose
 * node count (summed over the checkpoint's arrays) is >= T (default
 * T = SMs * max resident threads per SM, "the number of concurrent GPU
 * threads"), compares every node of l0, descends only below
 * unequal nodes and lists the unequal leaves: the potentially changed
 * chunks.  The result does not depend on T.
 *
 *   chunks      device, capacity `cap` uint64 chunk ids (global, ascending).
 *   n_chunks    (host) full count / (device) for the _async form.
 *   T           0 = default.
 * Errors: CKPT_EINVAL (NULL trees/outputs), CKPT_EMISMATCH (different
 * dtype, chunk_bytes, eps, array count or array lengths), CKPT_ETRUNC.
 * The _async form cannot report CKPT_ETRUNC (the count is on the device);
 * compare *n_chunks_dev with cap yourself.
 * ---------------------------------------------------------------------- */
ckpt_status ckpt_tree_diff(const ckpt_tree *a, const ckpt_tree *b, uint64_t *chunks, uint64_t cap,
                           uint64_t *n_chunks, void *stream);
ckpt_status ckpt_tree_diff_async(const ckpt_tree *a, const ckpt_tree *b, uint64_t T,
                                 uint64_t *chunks, uint64_t cap, uint64_t *n_chunks_dev,
                                 void *stream);

/* ------------------------------------------------------------------------
 * Step 4: stage-2 verification: for every listed chunk and
 * every element i in it, report i when fabs((double)a_i - (double)b_i) > eps
 * (binary64 for both dtypes, strict '>', NaN never differs; P:222,
 * P:713-716; R11).
 *
 *   a, b        device arrays of n elements (same layout as the build).
 *   chunks      device, ascending unique chunk ids (as produced by diff).
 *   n_chunks    (host) number of listed chunks.
 *   idx         device, capacity `cap` uint64 element ids (ascending).
 *   n_diff      (host) full count.
 * Errors: CKPT_EINVAL (NULL/misaligned pointers, bad chunk_bytes, eps < 0,
 * NaN or inf, chunk id out of range is NOT checked: ids must come from a
 * diff of trees of the same shape), CKPT_ETRUNC.
 * ---------------------------------------------------------------------- */
ckpt_status ckpt_verify(const void *a, const void *b, uint64_t n, ckpt_dtype dtype,
                        uint32_t chunk_bytes, const uint64_t *chunks, uint64_t n_chunks,
                        double eps, uint64_t *idx, uint64_t cap, uint64_t *n_diff, void *stream);

/* Multi-array, fully asynchronous form.  a, b, n are (host) arrays of
 * n_arrays entries.  The chunk count is read on the device from
 * *n_chunks_dev, clamped to chunks_cap; the full difference count is
 * written to *n_diff_dev (device). */
ckpt_status ckpt_verify_arrays_async(const void *const *a, const void *const *b, const uint64_t *n,
                                     uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                                     const uint64_t *chunks, const uint64_t *n_chunks_dev,
                                     uint64_t chunks_cap, double eps, uint64_t *idx, uint64_t cap,
                                     uint64_t *n_diff_dev, void *stream);

/* Steps 3+4 in one call on two trees and their arrays (a, b: host arrays of
 * the trees' n_arrays device pointers, same order and lengths as the build).
 * Writes the flagged chunk ids (as ckpt_tree_diff) and the differing element
 * ids (as ckpt_verify over those chunks) and counts_dev[0] / counts_dev[1]
 * (device) = their full counts.  The diff kernel(s) and the verify kernel
 * run back to back on `stream` with the chunk count kept on the device.
 * (A single fused kernel -- tile of leaves, verify its flagged chunks, two
 * look-backs -- was measured 1.5-3x slower: flagged chunks cluster, so
 * leaf-sized tiles serialise the verify work.)  Asynchronous. */
ckpt_status ckpt_diff_verify_async(const ckpt_tree *a, const ckpt_tree *b, const void *const *arrays_a,
                                   const void *const *arrays_b, uint64_t *chunks, uint64_t chunks_cap,
                                   uint64_t *idx, uint64_t idx_cap, uint64_t *counts_dev, void *stream);

/* ----------------------------------------------------------------------
 * Fused pair compare: steps 1-4 for two checkpoints of identical shape in
 * one call -- the device-resident form of the paper's online comparison
 * (SURVEY 8(f) rank 1).  One leaf-kernel launch hashes A and B
 * (Alg. 1); whichever warp finishes the second half of a 32-chunk
 * pair-task compares the two runs' leaf digests in-kernel and writes a flag
 * byte per chunk -- the BFS of P:555-566 at start level 0 (a chunk is flagged
 * iff its leaves differ), with no pass over the leaves afterwards.  The
 * flags are compacted into the ascending chunk list and the verify kernels
 * write the ascending element ids.  Both trees are built in full
 * (interior levels on a side stream, as ckpt_tree_build_batch) and returned
 * in *out_a / *out_b (owned by the caller, free with ckpt_tree_free).
 *   a, b        (host) arrays of n_arrays device pointers, 16-byte aligned
 *   n           (host) element counts, shared by A and B
 *   chunks      device, chunks_cap entries: flagged chunk ids, ascending
 *   idx         device, idx_cap entries: differing element ids (global
 *               numbering over the arrays in order), ascending
 *   counts_dev  device uint64[2]: full chunk count; element count over the
 *               listed (first chunks_cap) chunks
 * Results equal ckpt_tree_build_batch + ckpt_tree_diff + ckpt_verify (the
 * BFS finds the same chunks from any start level).  Scratch: one byte per
 * chunk plus the verify work buffer.  Errors: EINVAL, ENOMEM, ECUDA.
 * Asynchronous (no host synchronisation). */
ckpt_status ckpt_compare_pair_async(const void *const *a, const void *const *b, const uint64_t *n,
                                    uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                                    double eps, uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx,
                                    uint64_t idx_cap, uint64_t *counts_dev, void *stream,
                                    ckpt_tree **out_a, ckpt_tree **out_b);
/* Same with a hash block size (see ckpt_tree_build_batch_ex). */
ckpt_status ckpt_compare_pair_ex(const void *const *a, const void *const *b, const uint64_t *n,
                                 uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                                 double eps, uint32_t hash_block, uint64_t *chunks,
                                 uint64_t chunks_cap, uint64_t *idx, uint64_t idx_cap,
                                 uint64_t *counts_dev, void *stream, ckpt_tree **out_a,
                                 ckpt_tree **out_b);

/* ------------------------------------------------------------------------
 * One-call pair comparison (steps 1-4 on two checkpoints of n_arrays
 * arrays each), the library API of P:254-257.  Device inputs.  Writes the
 * chunk list and element ids to the caller's device buffers and both full
 * counts to (host) *n_chunks / *n_diff; root_a16 / root_b16 (host, may be
 * NULL) receive the two checkpoint roots.  Synchronises `stream`.
 * ---------------------------------------------------------------------- */
ckpt_status ckpt_compare(const void *const *a, const void *const *b, const uint64_t *n,
                         uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes, double eps,
                         uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx, uint64_t idx_cap,
                         uint64_t *n_chunks, uint64_t *n_diff, uint8_t *root_a16,
                         uint8_t *root_b16, void *stream);

/* Same with HOST inputs and outputs: a, b are (host) arrays of host
 * pointers (pinned memory is fastest; pageable works).  The library copies
 * both runs into one device staging allocation, runs steps 1-4 on the fused
 * pair path (ckpt_compare_pair_async), sizes the device element-id buffer to
 * the verified count (read back after the verify scan) and copies the ids
 * into idx (host, capacity idx_cap).  Synchronous.  Device memory used:
 * both runs + 8 bytes per chunk + 8 bytes per reported id; it stays cached in
 * the library's stream-ordered pool (see ckpt_trim_device_memory). */
ckpt_status ckpt_compare_host(const void *const *a, const void *const *b, const uint64_t *n,
                              uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                              double eps, uint64_t *idx, uint64_t idx_cap, uint64_t *n_chunks,
                              uint64_t *n_diff, uint8_t *root_a16, uint8_t *root_b16);

/* Out-of-core form: runs larger than HBM, or simply
 * host-resident, are streamed through a two-slot device ring of segments of
 * segment_bytes (rounded down to a multiple of chunk_bytes; a segment never
 * spans two arrays).  The H2D copy of segment k+1 (own stream) overlaps the
 * hashing (fused pair leaf kernel), compaction and verify of segment k, the
 * paper's I/O/compute overlap (Fig. 3) with PCIe in place
 * of Lustre.  Leaves land at their global position in full-size device trees,
 * so the roots equal the in-HBM build's; interior levels are built at the end.
 *   a, b        (host) arrays of n_arrays HOST pointers (pinned for full
 *               overlap; pageable works, with synchronous copies)
 *   hash_block  as ckpt_tree_build_batch_ex (16 = default)
 *   chunks, idx (host) outputs, capacities chunks_cap / idx_cap, ascending
 *               global ids; either may be NULL with capacity 0
 *   n_chunks, n_diff (host) full counts; root_a16 / root_b16 (host, may be
 *               NULL) the checkpoint roots
 * Device memory: 4 x segment_bytes + both trees (32 B per chunk each) + one
 * byte per chunk + the largest segment's ids.  Synchronous.  Errors as
 * ckpt_compare_host. */
ckpt_status ckpt_compare_stream(const void *const *a, const void *const *b, const uint64_t *n,
                                uint32_t n_arrays, ckpt_dtype dtype, uint32_t chunk_bytes,
                                double eps, uint32_t hash_block, uint64_t segment_bytes,
                                uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx,
                                uint64_t idx_cap, uint64_t *n_chunks, uint64_t *n_diff,
                                uint8_t *root_a16, uint8_t *root_b16);

/* ------------------------------------------------------------------------
 * Tree persistence.  The tree is built at capture time
 * and stored next to the checkpoint (metadata ~0.8% of the data
 * at 4 KB chunks); a later comparison loads it instead of re-hashing that run
 * and reads only the flagged chunks of the stored data (P:899-904,
 * P:1412-1416).
 *
 * Format (little-endian): "CKPTTRE1" | u32 version=1 | u32 dtype |
 * u32 chunk_bytes | u32 hash_block | f64 eps | u32 n_arrays | u32 0 |
 * u64 n_elems[n_arrays] | u64 node_count | 16-byte checkpoint root |
 * node_count x 16-byte nodes in the device layout (level-major across arrays,
 * then the top tree over the array roots; R13, R15).
 * ---------------------------------------------------------------------- */

/* (host) *bytes = size of the serialised tree.  CKPT_EINVAL for NULL or a
 * tree built from digests. */
ckpt_status ckpt_tree_serialized_size(const ckpt_tree *t, uint64_t *bytes);

/* Write the tree to dst (host, cap bytes; *written (host) = the size).  Waits
 * for the tree's levels and synchronises `stream`.  CKPT_EINVAL when cap is
 * smaller than ckpt_tree_serialized_size. */
ckpt_status ckpt_tree_serialize(const ckpt_tree *t, void *dst, uint64_t cap, uint64_t *written,
                                void *stream);

/* Load a serialised tree (src: host, `bytes` long) onto the current device.
 * The header is validated on the host before any device work: CKPT_EINVAL for
 * a bad magic/version, invalid parameters, a size that does not match the
 * header, or a stored root that differs from the last node.  Synchronises
 * `stream` (src may be reused on return).  The tree supports every tree
 * entry point (diff, roots, nodes, params, serialize). */
ckpt_status ckpt_tree_deserialize(const void *src, uint64_t bytes, void *stream, ckpt_tree **out);

/* Compare a live checkpoint (run B) with a stored run A: A's tree is loaded
 * from saved_a (host, saved_bytes; as ckpt_tree_deserialize), B's tree is
 * built with A's dtype / chunk_bytes / eps / hash_block, then steps 3+4 run
 * as ckpt_diff_verify_async.  a_data (host array of n_arrays pointers) are
 * run A's arrays: device pointers, or host memory the device can address
 * (pinned / registered, through unified addressing) -- the verify kernels
 * read only the flagged chunks of A.  b: device arrays; n (host): element
 * counts, which must equal the stored ones (else CKPT_EMISMATCH).  Outputs as
 * ckpt_compare_pair_async; both trees are returned (*out_a, *out_b).
 * Asynchronous after the tree upload. */
ckpt_status ckpt_compare_saved(const void *saved_a, uint64_t saved_bytes, const void *const *a_data,
                               const void *const *b, const uint64_t *n, uint32_t n_arrays,
                               uint64_t *chunks, uint64_t chunks_cap, uint64_t *idx,
                               uint64_t idx_cap, uint64_t *counts_dev, void *stream,
                               ckpt_tree **out_a, ckpt_tree **out_b);

/* ------------------------------------------------------------------------
 * Accessors (parity tests, multi-GPU driver)
 * ---------------------------------------------------------------------- */

/* Make `stream` wait until every level of the tree is built.  The library's
 * own entry points do this when they need interior nodes (K2 runs on an
 * internal side stream so that it overlaps a leaf-level diff and the
 * verify); call it before reading tree memory by other means, or to end a
 * timed region.  Asynchronous. */
ckpt_status ckpt_tree_wait(const ckpt_tree *t, void *stream);

/* (host outputs, any may be NULL) number of arrays, total leaves (= total
 * chunks), number of levels of the tallest array tree, total stored nodes
 * (all arrays, all levels; excludes the top tree over array roots). */
ckpt_status ckpt_tree_info(const ckpt_tree *t, uint32_t *n_arrays, uint64_t *n_leaves,
                           uint32_t *n_levels, uint64_t *n_nodes);

/* (host outputs, any may be NULL) the hashing parameters of a built tree:
 * dtype, chunk_bytes, eps and the effective hash block in bytes (16, ...,
 * chunk_bytes = whole chunk).  CKPT_EINVAL for trees built from digests. */
ckpt_status ckpt_tree_params(const ckpt_tree *t, ckpt_dtype *dtype, uint32_t *chunk_bytes,
                             double *eps, uint32_t *hash_block);

/* (host) 16-byte checkpoint root = root of the tree over the array roots
 * (equal to the array root when n_arrays == 1).  Synchronises `stream`. */
ckpt_status ckpt_tree_root(const ckpt_tree *t, uint8_t out16[16], void *stream);

/* Device copy of the n_arrays array roots (dst: device, n_arrays*16 bytes),
 * in array order.  Asynchronous. */
ckpt_status ckpt_tree_array_roots(const ckpt_tree *t, void *dst, void *stream);

/* Device copy of every node of array `array` (all levels, leaf-first, root
 * last; the oracle's layout) into dst (device, cap_bytes).  Asynchronous.
 * CKPT_EINVAL if array is out of range or cap_bytes is too small. */
ckpt_status ckpt_tree_nodes(const ckpt_tree *t, uint32_t array, void *dst, uint64_t cap_bytes,
                            void *stream);
/* Node count of array `array` (host). */
ckpt_status ckpt_tree_array_info(const ckpt_tree *t, uint32_t array, uint64_t *n_leaves,
                                 uint64_t *n_nodes);

/* The library allocates device memory from the device's default stream-ordered
 * pool and keeps freed blocks cached there (no re-mapping between calls).
 * This returns every unused cached block of the current device to the
 * driver (synchronises the device). */
ckpt_status ckpt_trim_device_memory(void);

/* Default BFS threshold T for the current device (SMs * max threads/SM). */
uint64_t ckpt_default_bfs_threshold(void);

/* Number of kernels this library has launched in this process (all entry
 * points, all threads) -- lets benchmarks report their own launch count. */
uint64_t ckpt_launch_count(void);

/* Kernel timing hook for benchmarks (CUDA events on the launching stream).
 * `mask` selects kernel families by bit: bit k enables family k (0 = leaf
 * hash K1, 1 = tree levels K2, 2 = diff K3, 3 = verify K4); 0 disables all.
 * Every launch of an enabled family is bracketed by two events (an event
 * between two kernels also ends their programmatic-launch overlap, so enable
 * only what is measured).  ckpt_profile_read synchronises those events and
 * returns the summed device time in milliseconds and the launch count of
 * family k since the last reset.  Off by default. */
void ckpt_profile_enable(int mask);
void ckpt_profile_reset(void);
ckpt_status ckpt_profile_read(int k, double *ms, uint64_t *launches);
/* Timeline of the recorded launches since the last reset: for record i,
 * out[3i] = kernel family, out[3i+1] / out[3i+2] = start / end in ms relative
 * to the first record's start (host, cap records).  *n_records (host) = the
 * number recorded.  Synchronises the recorded events. */
ckpt_status ckpt_profile_timeline(double *out, uint64_t cap, uint64_t *n_records);

const char *ckpt_strerror(ckpt_status s);
/* Thread-local detail of the last error returned on this thread. */
const char *ckpt_last_error(void);
/* ABI version: (major << 16) | minor. */
uint32_t ckpt_version(void);

#ifdef __cplusplus
}
#endif

#endif /* CKPT_H */
