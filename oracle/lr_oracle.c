/*
 * oracle/lr_oracle.c — CPU ORACLE for the list-ranking consumer (§V).
 *
 * TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).  Plain, single
 * threaded, sequential restatement; shares no code with the CUDA path.
 *
 *   or_lr_rank_seq : the definition — "find the distance of any node in a
 *                    list of n nodes from either end of the list" (§V);
 *                    R17: distance from the head, by walking the list.
 *   or_lr_run      : a sequential replica of the randomised algorithm the
 *                    GPU runs, in the paper's order: Phase I = Alg.3
 *                    ReduceList (FIS rounds), Phase II = Helman-JaJa
 *                    [10] splitter ranking of the reduced list, Phase III =
 *                    re-insertion of removed nodes ("the nodes removed in
 *                    step 1 are re-inserted to get the final ranks").
 *                    Random bits come from the oracle generator (gg_oracle.c),
 *                    so the FIS sets and the splitter set are checkable
 *                    bit-exactly; the final ranks must equal or_lr_rank_seq.
 *
 * Readings: R13 b(u) = bit 63 of the draw; R14 head and tail
 * are never removed; R15 stop once the active count <= ceil(n / floor(log2 n));
 * R16' walker = the node's slot in the stable, compacted active array and
 * draw = round index (walkers are active in a prefix of rounds, so every
 * active walker is at draw r in round r); R18 splitters = head plus nodes
 * whose draw (next epoch) is < 2^64/64.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

uint64_t or_walker_draw(uint64_t m, uint32_t l, uint32_t l0, uint64_t seed, uint64_t t,
                        uint64_t j, uint64_t *x, uint64_t *y);
int or_walker_init(uint64_t m, uint32_t l0, uint64_t seed, uint64_t t, uint64_t *x, uint64_t *y);

/* rank[v] = number of links from the head to v (head = 0).  Returns the
 * number of nodes reached (n for a proper list). */
int64_t or_lr_rank_seq(int64_t n, const int32_t *succ, int64_t head, int32_t *rank)
{
    int64_t v = head, r = 0;
    while (v >= 0 && r < n) {
        rank[v] = (int32_t)r;
        r++;
        v = succ[v];
    }
    return r;
}

static int64_t floor_log2(int64_t n)
{
    int64_t L = 0;
    while ((1ll << (L + 1)) <= n)
        L++;
    return L;
}

/*
 * Outputs (all length n unless noted):
 *   rank[v]           final rank (distance from head)
 *   removed_round[v]  round in which v left the list in Phase I, -1 if it survived
 *   is_splitter[v]    1 if v was a Phase II splitter
 *   info[0..3]        (int64) rounds, reduced size, splitter count, total draws
 * Returns 0, or -1 on allocation failure.
 */
int or_lr_run(uint64_t m, uint32_t l, uint32_t l0, uint64_t seed, int64_t n,
              const int32_t *succ_in, const int32_t *pred_in, int64_t head, int64_t max_rounds,
              int32_t *rank, int32_t *removed_round, int32_t *is_splitter, int64_t *info)
{
    int32_t *succ = malloc(sizeof(int32_t) * n);
    int32_t *pred = malloc(sizeof(int32_t) * n);
    int64_t *w = malloc(sizeof(int64_t) * n);          /* links from v to succ(v) */
    int32_t *rem_pred = malloc(sizeof(int32_t) * n);
    int64_t *rem_dist = malloc(sizeof(int64_t) * n);
    int32_t *active = malloc(sizeof(int32_t) * n);
    int32_t *next_active = malloc(sizeof(int32_t) * n);
    uint8_t *bit = malloc(n);
    uint64_t *wx = malloc(sizeof(uint64_t) * n);       /* walker state by slot */
    uint64_t *wy = malloc(sizeof(uint64_t) * n);
    if (!succ || !pred || !w || !rem_pred || !rem_dist || !active || !next_active || !bit ||
        !wx || !wy)
        return -1;
    memcpy(succ, succ_in, sizeof(int32_t) * n);
    memcpy(pred, pred_in, sizeof(int32_t) * n);
    int64_t tail = head;
    while (succ[tail] >= 0)
        tail = succ[tail];
    for (int64_t v = 0; v < n; v++) {
        w[v] = 1;
        removed_round[v] = -1;
        is_splitter[v] = 0;
        active[v] = (int32_t)v;   /* A_0 = node ids in order */
        or_walker_init(m, l0, seed, (uint64_t)v, &wx[v], &wy[v]);
    }
    int64_t A = n;
    const int64_t L = floor_log2(n) > 0 ? floor_log2(n) : 1;
    const int64_t target = (n + L - 1) / L;
    int64_t rounds = 0, draws = 0;

    /* ---- Phase I: Alg.3 ReduceList ---- */
    while (A > target && rounds < max_rounds) {
        const int64_t r = rounds;
        /* l.5-7: each node draws getnextrand(); b(u) = bit 63 */
        for (int64_t i = 0; i < A; i++) {
            int64_t u = active[i];
            uint64_t lab = or_walker_draw(m, l, l0, seed, (uint64_t)i, (uint64_t)r, &wx[i], &wy[i]);
            bit[u] = (uint8_t)(lab >> 63);
            draws++;
        }
        /* l.8-9: decide on the bits of this round, before any splice */
        uint8_t *remove = calloc((size_t)A, 1);
        for (int64_t i = 0; i < A; i++) {
            int64_t u = active[i];
            if (u == head || u == tail)
                continue;
            if (bit[u] == 1 && bit[pred[u]] == 0 && bit[succ[u]] == 0)
                remove[i] = 1;
        }
        /* l.10: remove with book-keeping: splice, remember (pred, distance) */
        for (int64_t i = 0; i < A; i++) {
            if (!remove[i])
                continue;
            int64_t u = active[i], p = pred[u], s = succ[u];
            rem_pred[u] = (int32_t)p;
            rem_dist[u] = w[p];
            w[p] += w[u];
            succ[p] = (int32_t)s;
            pred[s] = (int32_t)p;
            removed_round[u] = (int32_t)r;
        }
        int64_t k = 0;
        for (int64_t i = 0; i < A; i++) {
            if (!remove[i]) {
                next_active[k] = active[i];  /* stable compaction; slot k keeps walker k */
                k++;
            }
        }
        free(remove);
        memcpy(active, next_active, sizeof(int32_t) * k);
        A = k;
        rounds++;
    }

    /* ---- Phase II: Helman-JaJa on the reduced list ---- */
    /* splitters: head, plus active slots whose next draw is < 2^64/64 */
    int64_t nspl = 0;
    for (int64_t i = 0; i < A; i++) {
        int64_t v = active[i];
        uint64_t lab = or_walker_draw(m, l, l0, seed, (uint64_t)i, (uint64_t)rounds, &wx[i], &wy[i]);
        draws++;
        if (v == head || (lab >> 58) == 0) {
            is_splitter[v] = 1;
            nspl++;
        }
    }
    /* sublist walk: from each splitter to the next one, local offsets */
    int64_t *local = malloc(sizeof(int64_t) * n);
    int64_t *sub_of = malloc(sizeof(int64_t) * n);
    int64_t *sub_len = malloc(sizeof(int64_t) * n);
    int64_t *sub_next = malloc(sizeof(int64_t) * n);
    int64_t *prefix = malloc(sizeof(int64_t) * n);
    for (int64_t i = 0; i < A; i++) {
        int64_t s = active[i];
        if (!is_splitter[s])
            continue;
        int64_t v = s, off = 0;
        for (;;) {
            local[v] = off;
            sub_of[v] = s;
            off += w[v];
            int64_t nx = succ[v];
            if (nx < 0 || is_splitter[nx]) {
                sub_len[s] = off;
                sub_next[s] = nx;
                break;
            }
            v = nx;
        }
    }
    /* prefix over splitters, in list order from the head's sublist */
    int64_t acc = 0;
    for (int64_t s = head; s >= 0; s = sub_next[s]) {
        prefix[s] = acc;
        acc += sub_len[s];
    }
    /* fix-up */
    for (int64_t i = 0; i < A; i++) {
        int64_t v = active[i];
        rank[v] = (int32_t)(prefix[sub_of[v]] + local[v]);
    }
    /* ---- Phase III: re-insert in reverse round order ---- */
    for (int64_t r = rounds - 1; r >= 0; r--)
        for (int64_t u = 0; u < n; u++)
            if (removed_round[u] == r)
                rank[u] = (int32_t)(rank[rem_pred[u]] + rem_dist[u]);

    info[0] = rounds;
    info[1] = A;
    info[2] = nspl;
    info[3] = draws;
    free(local); free(sub_of); free(sub_len); free(sub_next); free(prefix);
    free(succ); free(pred); free(w); free(rem_pred); free(rem_dist); free(active);
    free(next_active); free(bit); free(wx); free(wy);
    return 0;
}
