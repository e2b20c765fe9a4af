// sharded.cuh -- the sharded (multi-GPU) exact selection driver (
// kernels: dist_kernels.cuh; collectives: comm.cuh).  Included by driver.cuh
// inside its anonymous namespace.
//
// One call enqueues, on the caller's stream, with no host round trip until
// the result hand-off:
//   init + sizes exchange (each rank's n_r)      -> N, k checked on the device
//   D sharded levels (dist_kernels.cuh)          -> 2 exchanges per level
//   gather of the survivors into G-element buffers -> 1 exchange
//   the single-GPU levels (enqueue_exact_levels) on the gathered buffer,
//     identical on every rank, then the result hand-off.
// Every decision (window hit / equality exit / miss, pass-through, the gather
// offsets) is taken on the device from exchanged counts, identically on every
// rank, so every rank enqueues the same sequence of collectives.  If the plan
// was too short (the survivors exceed G, or the tail needs one more level) the
// host enqueues the missing levels after the hand-off, as run_exact does.
constexpr int DIST_S = 4096;              // sample slots per sharded level (wide K1)

struct DistLayout {                       // c->d_dist, u64 slots
    static constexpr size_t sizes = 0;                                       // [SS_MAX_LEVELS + 1][16]
    static constexpr size_t sizes_send = sizes + (SS_MAX_LEVELS + 1) * DIST_MAX_RANKS;
    static constexpr size_t rows_send = sizes_send + DIST_MAX_RANKS;         // [16][DIST_REC]
    static constexpr size_t rows_recv = rows_send + DIST_MAX_RANKS * DIST_REC;
    static constexpr size_t keys_send = rows_recv + DIST_MAX_RANKS * DIST_REC;   // [MAX_S]
    static constexpr size_t keys_recv = keys_send + MAX_S;
    static constexpr size_t total = keys_recv + MAX_S;
};

inline u64 dist_gather_cap(const ss_context* c) { return (u64)1 << (c->cfg.shard_gather_log2 ? c->cfg.shard_gather_log2 : 20); }

inline double dist_window_frac(float z, int s) {
    return (2.0 * (z * 0.5 * std::sqrt((double)s) + 2.0) + 1.0) / s;
}

template <typename T>
ss_status run_sharded(ss_context* c, const T* d, u64 n_local, u64 k, void* h_result, cudaStream_t st) {
    typedef typename Traits<T>::Key K;
    ss_comm::ShardComm* comm = c->comm;
    if (!comm) return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_select_sharded: no communicator (ss_comm_init first)");
    const int P = comm->nranks(), R = comm->rank();
    if (P > DIST_MAX_RANKS) return fail(c, SS_ERR_INVALID_ARGUMENT, "ss_select_sharded: at most 16 ranks");
    const u64 G = dist_gather_cap(c);
    const int b = c->cfg.b_exact, bd = c->cfg.b_deep ? c->cfg.b_deep : b;
    const int s_deep = std::min(sample_size(c->cfg, bd), std::max(1024, bd));
    const u32 B = (u32)c->cfg.base_case;
    const float z = std::min(c->cfg.spec_z, 16.0f);   // (a window can never cover a whole sample of 4096)
    ss_status rc;
    if ((rc = ensure_small(c))) return rc;
    if (c->cfg.profile && (rc = prof_init(c))) return rc;
    c->launches = 0;
    c->d2h = 0;
    // workspace: ping-pong level buffers (a level's window plus its chunk
    // padding, or a copy of the shard, or a tail level), the gather buffers,
    // the exchange buffers, oracle bytes of the tail's levels
    // (a CTA pads its last output chunk; a chunk is at most 1/8 of the CTA's share)
    const u64 slack = (u64)c->sms * KW_MINB * 1024 + n_local / 8;
    const u64 cap_el = std::max<u64>(n_local, G) + slack;
    for (int i = 0; i < 2; ++i)
        if ((rc = grow(c, &c->d_buf[i], &c->cap_buf[i], cap_el * sizeof(T)))) return rc;
    if ((rc = grow(c, (void**)&c->d_oracles, &c->cap_oracles, G + 64))) return rc;
    if ((rc = grow(c, &c->d_gather[0], &c->cap_gather[0], G * sizeof(T)))) return rc;
    if ((rc = grow(c, &c->d_gather[1], &c->cap_gather[1], G * sizeof(T)))) return rc;
    if ((rc = grow(c, &c->d_dist, &c->cap_dist, DistLayout::total * sizeof(u64)))) return rc;
    u64* dd = reinterpret_cast<u64*>(c->d_dist);
    u64* sizes = dd + DistLayout::sizes;
    auto sizes_at = [&](int lev) { return sizes + (size_t)lev * DIST_MAX_RANKS; };
    K* ksend = reinterpret_cast<K*>(dd + DistLayout::keys_send);
    K* krecv = reinterpret_cast<K*>(dd + DistLayout::keys_recv);
    u64* rsend = dd + DistLayout::rows_send;
    u64* rrecv = dd + DistLayout::rows_recv;
    T* gsend = reinterpret_cast<T*>(c->d_gather[0]);
    T* grecv = reinterpret_cast<T*>(c->d_gather[1]);
    const int eb = (int)sizeof(K);
    auto exchange = [&](const void* send, void* recv, size_t count, int ebytes, cudaStream_t q) -> ss_status {
        std::string err;
        const ss_status r = comm->allreduce_sum(send, recv, count, ebytes, q, err);
        if (r) return fail(c, r, err);
        return SS_OK;
    };

    // The plan must be the same on every rank (every rank enqueues the same
    // collectives), so it is made from a number every rank knows: the size of
    // the union.  The first call after ss_comm_init exchanges the sizes and
    // reads N back (one host round trip); later calls plan with the N of the
    // previous call (published with its result) -- a different N only makes
    // a level a pass-through or adds one after the hand-off, identically on
    // every rank.
    CK(launch_pdl(init_kernel<T>, dim3(1), dim3(256), 0, st, c->d_ctl, (int)(SS_MAX_LEVELS + 1), c->d_totals,
                  (int)(SS_MAX_LEVELS * MAX_B), c->d_res, n_local, k, 0, d, 0, (u64)c->cfg.seed, (K*)nullptr, (void*)nullptr));
    CKLAUNCH("init_kernel");
    CK(launch_pdl(dist_sizes_kernel, dim3(1), dim3(32), 0, st, dd + DistLayout::sizes_send, P, R, n_local));
    CKLAUNCH("dist_sizes_kernel");
    if ((rc = exchange(dd + DistLayout::sizes_send, sizes_at(0), (size_t)P, 8, st))) return rc;   // exchange 0
    CK(launch_pdl(dist_check_kernel, dim3(1), dim3(32), 0, st, (const u64*)sizes_at(0), P, k, c->d_res));
    CKLAUNCH("dist_check_kernel");
    c->launches += 3;
    if (!c->dist_n_plan) {
        u64 hs[DIST_MAX_RANKS] = {};
        CK(cudaMemcpyAsync(hs, sizes_at(0), sizeof(u64) * P, cudaMemcpyDeviceToHost, st));
        CK(cudaStreamSynchronize(st));
        for (int q = 0; q < P; ++q) c->dist_n_plan += hs[q];
        c->d2h += (int64_t)(sizeof(u64) * P);
    }
    // plan: sharded levels until the expected survivors fit the gather buffer
    const double f = dist_window_frac(z, DIST_S);
    double est = (double)c->dist_n_plan;
    int D = 0;
    while (est > (double)G && D < 8) {
        est = est * f * 1.1 + (double)P * c->sms * 32.0;    // window + chunk padding
        ++D;
    }
    auto tail_levels = [&](double m) {
        int L = 0;
        while (m > (double)B && L < 8) {
            m = m * 1.5 / (L ? bd : b);
            ++L;
        }
        return L;
    };

    // one sharded level at index lev: input `in`, output c->d_buf[lev & 1]
    auto dist_level = [&](int lev, const T* in, cudaStream_t q) -> ss_status {
        ss_status r2;
        LevelCtl* ctl = c->d_ctl + lev;
        CK(launch_pdl(dist_sample_kernel<T>, dim3(DIST_S / 256), dim3(256), 0, q, in, ctl, c->d_res,
                      (const u64*)sizes_at(lev), P, R, DIST_S, (u64)c->cfg.seed, lev, G, ksend,
                      rsend));
        CKLAUNCH("dist_sample_kernel");
        if ((r2 = exchange(ksend, krecv, DIST_S, eb, q))) return r2;                  // exchange 1
        if ((r2 = launch_k1_wide<T>(c, in, lev, DIST_S, 0u, q, krecv))) return r2;    // identical sorted sample
        CountArgs w{};
        w.ctl = ctl;
        w.ctl_next = c->d_ctl + lev + 1;
        w.res = c->d_res;
        w.sorted = reinterpret_cast<K*>(c->d_sorted) + (size_t)lev * MAX_S;
        w.s = DIST_S;
        w.spec_min_n = 0;
        w.spec_z = z;
        w.spec_max_frac = 1.0f;
        w.level = lev;
        w.tail = TAIL_EXACT;
        w.cap_out = c->d_buf[lev & 1];
        w.rec = rsend + (size_t)R * DIST_REC;
        mark(c, lev, 1, 0, q);
        if ((r2 = launch_window<T>(c, 0, in, w, q))) return r2;
        mark(c, lev, 1, 1, q);                     // profile 1/2: the level's fused kernel
        if ((r2 = exchange(rsend, rrecv, (size_t)P * DIST_REC, 8, q))) return r2;    // exchange 2
        CK(launch_pdl(dist_decide_kernel<T>, dim3(1), dim3(32), 0, q, ctl, c->d_ctl + lev + 1, c->d_res,
                      (const u64*)rrecv, P, R, sizes_at(lev + 1), lev));
        CKLAUNCH("dist_decide_kernel");
        CK(launch_pdl(dist_copy_kernel<T>, dim3((u32)c->sms * 4), dim3(256), 0, q, in,
                      reinterpret_cast<T*>(c->d_buf[lev & 1]), (const LevelCtl*)ctl, (const SelectResult*)c->d_res));
        CKLAUNCH("dist_copy_kernel");
        c->launches += 5;
        return SS_OK;
    };
    // sharded levels [lev0, lev_end), the gather at lev_end, the tail from
    // lev_end + 1 (L_tail levels, then the final K1)
    ExactPlan plan{};
    plan.b0 = b;
    plan.bd = bd;
    plan.s = s_deep;
    plan.s_deep = s_deep;
    plan.B = B;
    plan.sample0 = nullptr;
    auto enqueue = [&](int lev0, int lev_end, int L_tail, cudaStream_t q) -> ss_status {
        ss_status r2;
        const T* in = lev0 ? reinterpret_cast<const T*>(c->d_buf[(lev0 - 1) & 1]) : d;
        for (int lev = lev0; lev < lev_end; ++lev) {
            if ((r2 = dist_level(lev, in, q))) return r2;
            in = reinterpret_cast<const T*>(c->d_buf[lev & 1]);
        }
        CK(launch_pdl(dist_gather_kernel<T>, dim3((u32)c->sms * 4), dim3(256), 0, q, in,
                      (const LevelCtl*)(c->d_ctl + lev_end), c->d_ctl + lev_end + 1, c->d_res,
                      (const u64*)sizes_at(lev_end), P, R, G, gsend, lev_end));
        CKLAUNCH("dist_gather_kernel");
        ++c->launches;
        const int eg = sizeof(T) == 8 ? 8 : 4;
        if ((r2 = exchange(gsend, grecv, (size_t)G, eg, q))) return r2;               // exchange 3
        plan.lev_first = lev_end + 1;
        plan.L = lev_end + 1 + L_tail;
        return enqueue_exact_levels<T>(c, plan, grecv, lev_end + 1, q);
    };

    int L_tail = tail_levels(est);
    if (D + 1 + L_tail >= SS_MAX_LEVELS - 2) return fail(c, SS_ERR_INTERNAL, "sharded plan too deep");
    if ((rc = enqueue(0, D, L_tail, st))) return rc;
    if ((rc = enqueue_publish(c, st))) return rc;
    if ((rc = wait_publish(c, st))) return rc;
    int extra = 0;
    for (;;) {
        const SelectResult& h = *c->h_res;
        if (h.dist_halt == 2) return fail(c, SS_ERR_INVALID_ARGUMENT, "k must be in [0, total elements of all ranks)");
        if (h.dist_halt == 1) {                  // survivors exceed G: one more sharded level (every rank)
            if (D + 2 + L_tail >= SS_MAX_LEVELS - 2) return fail(c, SS_ERR_INTERNAL, "sharded recursion too deep");
            CK(cudaMemsetAsync(&c->d_res->done, 0, sizeof(int), st));
            CK(cudaMemsetAsync(&c->d_res->dist_halt, 0, sizeof(int), st));
            if ((rc = enqueue(D, D + 1, L_tail, st))) return rc;
            ++D;
        } else if (!h.done) {                    // the tail needs one more level
            if (!h.incomplete || D + 2 + L_tail >= SS_MAX_LEVELS - 2)
                return fail(c, SS_ERR_INTERNAL, "sharded recursion did not terminate");
            CK(cudaMemsetAsync(&c->d_res->incomplete, 0, sizeof(int), st));
            plan.lev_first = D + 1;
            plan.L = D + 2 + L_tail;
            if ((rc = enqueue_exact_levels<T>(c, plan, grecv, D + 1 + L_tail, st))) return rc;
            ++L_tail;
        } else {
            break;
        }
        if ((rc = enqueue_publish(c, st))) return rc;
        if ((rc = wait_publish(c, st))) return rc;
        ++extra;
    }
    const SelectResult& r = *c->h_res;
    c->dist_n_plan = r.dist_n;                 // the next call's plan (identical on every rank)
    std::memcpy(h_result, &r.bits, sizeof(T));
    ss_stats& S = c->stats;
    std::memset(&S, 0, sizeof(S));
    S.levels = r.levels;
    S.equality_exit = r.eq_exit;
    S.spec_levels = (int32_t)r.spec_levels;
    S.fused_levels = (int32_t)r.fused_levels;
    S.incomplete_rounds = extra;
    S.shard_levels = D;
    S.shard_ranks = P;
    for (int l = 0; l < SS_MAX_LEVELS; ++l) {
        S.n_level[l] = r.n_level[l];
        S.bucket[l] = r.bucket[l];
    }
    // algorithmic bytes summed over the ranks: each sharded level reads the
    // level once and writes its window (+ a copy on a miss); the gather writes
    // and receives the survivors on every rank; the tail (replicated on every
    // rank) follows the single-GPU byte model
    const double Sz = (double)sizeof(T);
    double bytes = 0;
    const int last_dist = std::min(D, r.levels);
    for (int l = 0; l < last_dist && !(r.eq_exit && l == r.levels - 1 && l < D); ++l) {
        const double nl = (double)r.n_level[l], nn = (double)r.n_level[l + 1];
        bytes += Sz * nl + ((r.fused_levels >> l & 1) ? Sz * nn : 2.0 * Sz * nl);
    }
    if (!r.eq_exit || r.levels > D) {
        const double ng = (double)r.n_level[D];
        bytes += Sz * ng * (1.0 + P);            // each rank writes its part, every rank receives all
        for (int l = D + 1; l < r.levels; ++l) {
            const double nl = (double)r.n_level[l], nn = (double)r.n_level[l + 1];
            const bool last_eq = r.eq_exit && l == r.levels - 1;
            bytes += P * (Sz * nl + nl + (last_eq ? 0.0 : nl + 2.0 * Sz * nn));
        }
        if (!r.eq_exit) bytes += P * Sz * (double)r.n_level[r.levels];
    }
    S.bytes_algorithmic = bytes;
    S.launches = c->launches;
    S.d2h_bytes = c->d2h;
    c->launches_total += c->launches;
    c->calls_total += 1;
    prof_collect(c);
    return SS_OK;
}
