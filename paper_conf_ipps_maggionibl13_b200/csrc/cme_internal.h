// Internal declarations of libcme (not part of the ABI; see include/cme.h).
#pragma once

#include <cstdint>
#include <string>
#include <vector>

#include "cme.h"
#include "comm.h"

namespace cme {

// Thread-local error detail for cme_last_error().
void set_error(const std::string& msg);

// Off-diagonal part of A by rows (row i <- col j: transition j -> i) + diagonal.
// A batch of B rate sets shares the pattern: values are member-minor
// (v[p*B + b], d[i*B + b]); B = 1 is the ordinary single matrix.
struct Csr {
    int64_t n = 0;
    int32_t B = 1;
    std::vector<int64_t> rp;   // n + 1
    std::vector<int32_t> ci;   // column indices, ascending within a row
    std::vector<double> v;     // rates, nnz * B
    std::vector<double> d;     // a_ii (< 0), n * B
    int64_t nnz() const { return rp.empty() ? 0 : rp.back(); }
};

// Ingest of B rate sets rate[b*nnz + e] on one COO pattern.
cme_status ingest_coo(int64_t n, int64_t nnz, const int32_t* row, const int32_t* col,
                      const double* rate, int32_t B, uint32_t flags, Csr& out);

// Orderings and graph tests (R1, R11, R12).
void order_dfs(const Csr& A, int64_t root, std::vector<int32_t>& new_to_old);
void order_rcm(const Csr& A, std::vector<int32_t>& new_to_old);
int64_t directed_period(const Csr& A, int64_t root);
void permute(const Csr& A, const std::vector<int32_t>& new_to_old, Csr& out);

// Packed layout v0 ("DIAG + warp-grained SELL") of rows
// [r0, r1) of an ordered matrix, columns shifted by -col_shift.
struct Packed {
    int64_t n = 0, n_slots = 0, n_slices = 0, n_ell = 0;
    int32_t band_on = 0, window = 1, group = 1, B = 1;
    std::vector<double> lo, up, inv_d;    // slot order, n_slots * B (member-minor)
    std::vector<double> dneg;             // slot order: -A_rr (0 for pad slots), for the compact encoding
    std::vector<int32_t> row_of;          // slot -> local row
    std::vector<int64_t> slice_off;       // n_slices + 1
    std::vector<int32_t> slice_w;         // n_slices
    std::vector<double> val;              // n_ell * B (member-minor)
    std::vector<int32_t> col;             // n_ell (shared by the batch)
    // CSR arm
    std::vector<int64_t> csr_rp;
    std::vector<int32_t> csr_ci;
    std::vector<double> csr_v;
};
bool band_rule(const Csr& A, int band_mode);
// group: slices sharing one width (1 warp-grained, 8 block-sliced, 0 = global ELL width)
void pack_rows(const Csr& A, int64_t r0, int64_t r1, int64_t col_shift, int32_t window,
               bool band_on, int32_t group, int32_t global_kmax, Packed& P);
void pack_csr_rows(const Csr& A, int64_t r0, int64_t r1, int64_t col_shift, Packed& P);

// Compact encoding of a B = 1 layout-v0 pack: the rows of
// M = |D|^-1 O instead of O + inv_d (val_c = a_rj / (-a_rr), lo/up likewise),
// 16-bit column offsets relative to the row (col16 = j - r), 8-bit row offsets
// inside the rearrangement window (row8 = r - window base).  Returns false
// (and leaves C empty) when the pack does not qualify: batch, a window that is
// not a power of two <= 256, or an offset outside int16.  own_off: x-span
// index of local row 0 (the column coordinates of P.col).
struct Compact {
    bool valid = false;                   // encoded
    int32_t win_shift = 0;                // log2(window), 0 = no rearrangement
    std::vector<double> val, lo, up;      // val: n_ell; lo/up: n_slots (band only)
    std::vector<int16_t> col16;           // n_ell
    std::vector<uint8_t> row8;            // n_slots (rearranged packs only)
    // value-indexed variant (CSR-VI style): the distinct stored values of O
    // (val entries incl. pads, lo/up when the band is on) -- for a batch the
    // distinct B-tuples, shared indices -- ascending, and 16-bit indices into
    // that dictionary; inv_d stays per row (and member).  A batch's Compact
    // holds only the offsets (col16, row8) besides the value index.
    bool vi_valid = false;
    std::vector<double> dict;             // <= 65536 tuples x B, ascending (lexicographic), member-minor
    std::vector<uint16_t> vidx;           // n_ell
    std::vector<uint16_t> loi, upi;       // n_slots (band only)
};
bool encode_compact(const Packed& P, int64_t own_off, Compact& C);
// Value-index P's layout-v0 values into C (needs C.valid); false when the
// pack holds more than 65536 distinct values.
bool encode_value_index(const Packed& P, Compact& C);
// x-window plan (device.cu): per tile of ts slices the
// monotone chunk range [ch.x, ch.y) of 256-row iterate chunks (chunk k = rows
// [256 k - xoff, 256 k - xoff + 256)); xw_need = ring chunks with S stages in
// flight, span = the widest tile's chunk count.
void xw_plan(const Packed& P, int ts, bool band, int64_t own_off, int xoff, int64_t nx, std::vector<int2>& ch);
int64_t xw_need(const std::vector<int2>& ch, int S, int64_t& span);

struct Device;  // device state (device.cu)

}  // namespace cme

struct cme_comm_s;

struct cme_matrix_s {
    int stage = 0;              // 1 created, 2 packed, 3 distributed
    cme::Csr A;                 // original order
    int order = CME_ORDER_NONE;
    std::vector<int32_t> perm;  // new_to_old
    cme::Csr B;                 // reordered (valid after pack)
    int format = CME_FMT_DIAG_SELL;
    cme_pack_opts popts{32, 256, CME_BAND_AUTO, -1};
    bool band_on = false;
    int64_t period = 0;
    std::vector<double> norm_inf;  // ||A_b||_inf per batch member
    cme::Packed P;              // local packed layout (whole matrix unless distributed)
    cme::Compact Cpt;           // its compact encoding when the device uses it (else empty)
    int32_t global_kmax = 0;
    cme_solver_opts sopts{0.0, 100, CME_STOP_DELTA_L1, 1e-10, nullptr};
    cme_report report{};
    std::vector<cme_report> member_reports;  // per batch member
    // partition
    int nranks = 1, rank = 0;
    std::vector<int64_t> cuts;  // nranks + 1
    std::vector<int64_t> span;  // 2 * nranks
    cme::HaloPlan halo;         // this rank's exchange plan
    std::vector<int32_t> halo_speer, halo_rpeer;
    cme_comm_s* comm = nullptr;
    cme::Device* dev = nullptr;
};

// Enumerated network (cme_network_enumerate / cme_network_enumerate_gpu).
struct cme_coo_s {
    int64_t n = 0, nnz = 0;
    int32_t m = 0;
    std::vector<int32_t> states, row, col;
    std::vector<double> rate;
};
