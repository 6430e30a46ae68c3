/*
 * ksel_oracle.c -- CPU ORACLE for batched k-selection and brute-force k-NN.
 *
 * TEST INFRASTRUCTURE ONLY.  Nothing in the product path (the CUDA library
 * libksel.so or the Python binding paper_conf_ipps_tang0emg15_b200/) may
 * include, link, call or execute this file.  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs use it.  It shares no
 * code, headers, tables or helpers with csrc/.
 *
 * It is deliberately plain and slow: the result is the *definition* of the
 * selection written out, not an algorithm from the paper.  The paper's methods
 * (Merge Queue, Buffered Search, Hierarchical Partition) all reach exactly the
 * k smallest elements:
 *   - PAPER.md L11 (Sec. I): "finding the k smallest values from a given
 *     unordered list of distances, which is called k-selection";
 *   - PAPER.md L19 (Algorithm 1): scan (dist, id), insert when
 *     dist < dqueue[0] (strict <, in index order => among equal values the
 *     lower index is kept);
 *   - PAPER.md L225 (Sec. III.E): HP "guarantees that the k smallest elements
 *     will be contained in the queue";
 *   - PAPER.md L637 (Sec. V): the output is expected sorted (QMS is faulted for
 *     unsorted output).
 * So for each row: form (value, index) pairs, sort them by the total order
 * "value, then index", keep the first k.  Readings:
 *   R1 ties -> lower index first; R2 output ascending; R3 -0.0 == +0.0;
 *   R4 NaN greater than +Inf, all NaNs equal; R5 +-Inf and denormals are
 *   ordinary values; R8 int32 0-based indices; R9 squared L2, no sqrt.
 *
 * Pinned by tests/test_oracle_pins.py (brute-force rank counting over an
 * exhaustive tiny alphabet, numpy stable argsort, invariants, the paper's
 * worked examples in tests/golden/).
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

typedef struct {
    float v;
    int32_t i;
} pair_t;

/* Value order of readings R3-R5: IEEE "<" for non-NaN values (so -0.0 == +0.0),
 * every NaN after every non-NaN value, NaNs equal to each other. */
static int value_less(float a, float b) {
    int an = isnan(a), bn = isnan(b);
    if (an) return 0;
    if (bn) return 1;
    return a < b;
}

/* Total order "(value, index)" (reading R1: ties by lower index). */
static int pair_cmp(const void* pa, const void* pb) {
    const pair_t* a = (const pair_t*)pa;
    const pair_t* b = (const pair_t*)pb;
    if (value_less(a->v, b->v)) return -1;
    if (value_less(b->v, a->v)) return 1;
    return (a->i > b->i) - (a->i < b->i);
}

/* One row: pairs (dist[j], j), sort, first k.  Any correct sort gives the same
 * result because pair_cmp is a total order on distinct indices. */
static void select_row(const float* row, int64_t N, int64_t k, pair_t* scratch,
                       float* out_val, int32_t* out_idx) {
    for (int64_t j = 0; j < N; ++j) {
        scratch[j].v = row[j];
        scratch[j].i = (int32_t)j;
    }
    qsort(scratch, (size_t)N, sizeof(pair_t), pair_cmp);
    for (int64_t t = 0; t < k; ++t) {
        out_val[t] = scratch[t].v; /* bit copy of the input value */
        out_idx[t] = scratch[t].i;
    }
}

typedef struct {
    const float* dist;
    int64_t Q, N, k;
    float* out_val;
    int32_t* out_idx;
    int64_t r0, r1;
    int err;
} select_job_t;

static void* select_worker(void* arg) {
    select_job_t* j = (select_job_t*)arg;
    pair_t* scratch = (pair_t*)malloc(sizeof(pair_t) * (size_t)(j->N > 0 ? j->N : 1));
    if (!scratch) { j->err = 1; return NULL; }
    for (int64_t r = j->r0; r < j->r1; ++r)
        select_row(j->dist + r * j->N, j->N, j->k, scratch, j->out_val + r * j->k,
                   j->out_idx + r * j->k);
    free(scratch);
    return NULL;
}

/* Run fn on n jobs (each job_size bytes) with one POSIX thread per job. */
static int spawn(void* (*fn)(void*), void* jobs, size_t job_size, int n) {
    pthread_t* th = (pthread_t*)malloc(sizeof(pthread_t) * (size_t)n);
    if (!th) return 1;
    int err = 0, started = 0;
    for (int t = 0; t < n; ++t) {
        if (pthread_create(&th[t], NULL, fn, (char*)jobs + (size_t)t * job_size) != 0) { err = 1; break; }
        ++started;
    }
    for (int t = 0; t < started; ++t) pthread_join(th[t], NULL);
    free(th);
    return err;
}

static int clamp_threads(int nthreads, int64_t Q) {
    if (nthreads < 1) nthreads = 1;
    if (nthreads > Q) nthreads = (int)Q;
    return nthreads;
}

/* oracle_select: out[q][0..k) = the k smallest (dist[q][j], j) in the total
 * order above, ascending.  dist is Q x N row-major (host).  Any 1 <= k <= N.
 * Returns 0 on success, nonzero on bad arguments / allocation failure. */
int oracle_select(const float* dist, int64_t Q, int64_t N, int64_t k, float* out_val,
                  int32_t* out_idx, int nthreads) {
    if (!dist || !out_val || !out_idx || Q < 0 || N < 1 || k < 1 || k > N) return 2;
    if (Q == 0) return 0;
    nthreads = clamp_threads(nthreads, Q);
    select_job_t* jobs = (select_job_t*)calloc((size_t)nthreads, sizeof(select_job_t));
    if (!jobs) return 1;
    for (int t = 0; t < nthreads; ++t) {
        jobs[t].dist = dist; jobs[t].Q = Q; jobs[t].N = N; jobs[t].k = k;
        jobs[t].out_val = out_val; jobs[t].out_idx = out_idx;
        jobs[t].r0 = Q * t / nthreads; jobs[t].r1 = Q * (t + 1) / nthreads;
    }
    int err = spawn(select_worker, jobs, sizeof(select_job_t), nthreads);
    for (int t = 0; t < nthreads && !err; ++t) err |= jobs[t].err;
    free(jobs);
    return err;
}

/* oracle_merge: cand_val/cand_idx are [S][Q][kin] (S candidate lists per query,
 * explicit indices).  out[q] = the k smallest (value, index) pairs of the union
 * of the S lists, ascending -- "divide-and-merge" (ref. [18]).
 * Written as: concatenate, sort by the same total order, truncate. */
int oracle_merge(const float* cand_val, const int32_t* cand_idx, int64_t Q, int64_t S,
                 int64_t kin, int64_t k, float* out_val, int32_t* out_idx) {
    if (!cand_val || !cand_idx || !out_val || !out_idx || Q < 0 || S < 1 || kin < 1 || k < 1 ||
        k > S * kin)
        return 2;
    pair_t* scratch = (pair_t*)malloc(sizeof(pair_t) * (size_t)(S * kin));
    if (!scratch) return 1;
    for (int64_t q = 0; q < Q; ++q) {
        int64_t n = 0;
        for (int64_t s = 0; s < S; ++s)
            for (int64_t t = 0; t < kin; ++t) {
                scratch[n].v = cand_val[(s * Q + q) * kin + t];
                scratch[n].i = cand_idx[(s * Q + q) * kin + t];
                ++n;
            }
        qsort(scratch, (size_t)n, sizeof(pair_t), pair_cmp);
        for (int64_t t = 0; t < k; ++t) {
            out_val[q * k + t] = scratch[t].v;
            out_idx[q * k + t] = scratch[t].i;
        }
    }
    free(scratch);
    return 0;
}

/* oracle_knn_dist: the Euclidean-distance phase (Sec. II.A),
 * reading R9: squared L2, no sqrt.  Naive triple loop, every term in double,
 * one rounding to fp32 at the end:
 *   out[q][r] = (float) sum_{t<D} ((double)query[q][t] - (double)ref[r][t])^2
 * ref is N x D, query is Q x D, out is Q x N (row-major, host). */
typedef struct {
    const float *ref, *query;
    int64_t N, Q, D;
    float* out;
    int64_t r0, r1;
} dist_job_t;

static void* dist_worker(void* arg) {
    dist_job_t* j = (dist_job_t*)arg;
    for (int64_t q = j->r0; q < j->r1; ++q)
        for (int64_t r = 0; r < j->N; ++r) {
            double acc = 0.0;
            for (int64_t t = 0; t < j->D; ++t) {
                double d = (double)j->query[q * j->D + t] - (double)j->ref[r * j->D + t];
                acc += d * d;
            }
            j->out[q * j->N + r] = (float)acc;
        }
    return NULL;
}

int oracle_knn_dist(const float* ref, const float* query, int64_t N, int64_t Q, int64_t D,
                    float* out, int nthreads) {
    if (!ref || !query || !out || N < 1 || Q < 0 || D < 1) return 2;
    if (Q == 0) return 0;
    nthreads = clamp_threads(nthreads, Q);
    dist_job_t* jobs = (dist_job_t*)calloc((size_t)nthreads, sizeof(dist_job_t));
    if (!jobs) return 1;
    for (int t = 0; t < nthreads; ++t) {
        jobs[t].ref = ref; jobs[t].query = query; jobs[t].N = N; jobs[t].Q = Q;
        jobs[t].D = D; jobs[t].out = out;
        jobs[t].r0 = Q * t / nthreads; jobs[t].r1 = Q * (t + 1) / nthreads;
    }
    int err = spawn(dist_worker, jobs, sizeof(dist_job_t), nthreads);
    free(jobs);
    return err;
}

/* oracle_knn: distances as above, then oracle_select on each query row with
 * indices shifted by idx_offset (global reference ids for row-sharded runs).
 * scratch_dist must hold Q*N floats. */
int oracle_knn(const float* ref, const float* query, int64_t N, int64_t Q, int64_t D, int64_t k,
               int64_t idx_offset, float* scratch_dist, float* out_dist, int32_t* out_idx,
               int nthreads) {
    int err = oracle_knn_dist(ref, query, N, Q, D, scratch_dist, nthreads);
    if (err) return err;
    err = oracle_select(scratch_dist, Q, N, k, out_dist, out_idx, nthreads);
    if (err) return err;
    for (int64_t t = 0; t < Q * k; ++t) out_idx[t] = (int32_t)(out_idx[t] + idx_offset);
    return 0;
}

/* oracle_knn_graph: the k-nearest-neighbour graph of one point set (the k-NNG
 * construction QMS [9] targets): for every point
 * i of points[N][D], the k smallest (d(i, j), j) over j != i -- distances as in
 * oracle_knn_dist, order as in oracle_select.  Definition, written out: the
 * pairs of row i without j == i, sorted, first k.  Requires 1 <= k <= N - 1.
 * scratch_dist must hold N*N floats. */
int oracle_knn_graph(const float* points, int64_t N, int64_t D, int64_t k, float* scratch_dist,
                     float* out_dist, int32_t* out_idx, int nthreads) {
    if (!points || !scratch_dist || !out_dist || !out_idx || N < 2 || k < 1 || k > N - 1) return 2;
    int err = oracle_knn_dist(points, points, N, N, D, scratch_dist, nthreads);
    if (err) return err;
    pair_t* scratch = (pair_t*)malloc(sizeof(pair_t) * (size_t)N);
    if (!scratch) return 1;
    for (int64_t i = 0; i < N; ++i) {
        int64_t n = 0;
        for (int64_t j = 0; j < N; ++j) {
            if (j == i) continue;
            scratch[n].v = scratch_dist[i * N + j];
            scratch[n].i = (int32_t)j;
            ++n;
        }
        qsort(scratch, (size_t)n, sizeof(pair_t), pair_cmp);
        for (int64_t t = 0; t < k; ++t) {
            out_dist[i * k + t] = scratch[t].v;
            out_idx[i * k + t] = scratch[t].i;
        }
    }
    free(scratch);
    return 0;
}
