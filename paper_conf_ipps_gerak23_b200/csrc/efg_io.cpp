// efg_io.cpp — on-disk EFG (efg_save / efg_load): a built graph written once
// and loaded without rebuilding (SURVEY §5 checkpoint row).  The file is the
// P:113 arrays (vlist, num_lower_bits, offsets, data) plus what the builder
// derives from them for the traversal (largest neighbour, in-edge flags, the
// degree relabelling, CSR-order weights), after a fixed header that states
// every array's length.  Native byte order; the header's magic and version
// guard the format.
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "efg_internal.h"

namespace efg {
namespace {

constexpr char kMagic[8] = {'E', 'F', 'G', 'R', 'A', 'P', 'H', '1'};
constexpr uint32_t kVersion = 1;

struct FileHeader {
    char magic[8];
    uint32_t version;
    uint32_t k;
    uint64_t n, m, m_input, row_lo, row_hi;
    uint64_t symmetric;
    uint64_t fwd_bytes, lower_bytes, upper_bytes, apriori_bits;
    // element counts: vlist, nlb, offsets, data, umax, has_in, old_of_new, new_of_old, weights
    uint64_t count[9];
    uint64_t reserved[4];
};

struct File {
    FILE *f = nullptr;
    ~File()
    {
        if (f) std::fclose(f);
    }
};

template <class T>
bool write_vec(FILE *f, const std::vector<T> &v)
{
    return v.empty() || std::fwrite(v.data(), sizeof(T), v.size(), f) == v.size();
}

template <class T>
bool read_vec(FILE *f, std::vector<T> &v, uint64_t count)
{
    try {
        v.resize(count);
    } catch (...) {
        return false;
    }
    return count == 0 || std::fread(v.data(), sizeof(T), count, f) == count;
}

}  // namespace

efg_status save_host(const HostEFG &h, const char *path)
{
    File fh;
    fh.f = std::fopen(path, "wb");
    if (!fh.f) return set_error(EFG_EIO, std::string("efg_save: cannot open ") + path + " for writing");
    FileHeader hd;
    std::memset(&hd, 0, sizeof(hd));
    std::memcpy(hd.magic, kMagic, sizeof(kMagic));
    hd.version = kVersion;
    hd.k = h.k;
    hd.n = h.n;
    hd.m = h.m;
    hd.m_input = h.m_input;
    hd.row_lo = h.row_lo;
    hd.row_hi = h.row_hi;
    hd.symmetric = h.symmetric ? 1 : 0;
    hd.fwd_bytes = h.fwd_bytes;
    hd.lower_bytes = h.lower_bytes;
    hd.upper_bytes = h.upper_bytes;
    hd.apriori_bits = h.apriori_bits;
    const uint64_t c[9] = {h.vlist.size(), h.nlb.size(), h.offsets.size(), h.data.size(), h.umax.size(),
                           h.has_in.size(), h.old_of_new.size(), h.new_of_old.size(), h.weights.size()};
    std::memcpy(hd.count, c, sizeof(c));
    bool ok = std::fwrite(&hd, sizeof(hd), 1, fh.f) == 1;
    ok = ok && write_vec(fh.f, h.vlist) && write_vec(fh.f, h.nlb) && write_vec(fh.f, h.offsets) &&
         write_vec(fh.f, h.data) && write_vec(fh.f, h.umax) && write_vec(fh.f, h.has_in) &&
         write_vec(fh.f, h.old_of_new) && write_vec(fh.f, h.new_of_old) && write_vec(fh.f, h.weights);
    ok = std::fflush(fh.f) == 0 && ok;
    if (!ok) return set_error(EFG_EIO, std::string("efg_save: write to ") + path + " failed");
    return EFG_OK;
}

efg_status load_host(const char *path, HostEFG &h)
{
    File fh;
    fh.f = std::fopen(path, "rb");
    if (!fh.f) return set_error(EFG_EIO, std::string("efg_load: cannot open ") + path);
    FileHeader hd;
    if (std::fread(&hd, sizeof(hd), 1, fh.f) != 1 || std::memcmp(hd.magic, kMagic, sizeof(kMagic)) != 0)
        return set_error(EFG_EIO, std::string("efg_load: ") + path + " is not an EFG file");
    if (hd.version != kVersion) return set_error(EFG_EIO, "efg_load: unsupported EFG file version");
    const uint64_t *c = hd.count;
    // the shapes the builder produces (a row-range handle keeps full-length vertex arrays)
    const bool shape = hd.n >= 1 && hd.n <= 0xFFFFFFFFull && c[0] == hd.n + 1 && c[1] == hd.n &&
                       c[2] == hd.n + 1 && c[4] == hd.n && (c[5] == 0 || c[5] == hd.n) && c[6] == c[7] &&
                       (c[6] == 0 || c[6] == hd.n) && (c[8] == 0 || c[8] == hd.m) && hd.row_hi <= hd.n &&
                       hd.row_lo <= hd.row_hi;
    if (!shape) return set_error(EFG_EIO, "efg_load: inconsistent EFG file header");
    bool ok = read_vec(fh.f, h.vlist, c[0]) && read_vec(fh.f, h.nlb, c[1]) && read_vec(fh.f, h.offsets, c[2]) &&
              read_vec(fh.f, h.data, c[3]) && read_vec(fh.f, h.umax, c[4]) && read_vec(fh.f, h.has_in, c[5]) &&
              read_vec(fh.f, h.old_of_new, c[6]) && read_vec(fh.f, h.new_of_old, c[7]) &&
              read_vec(fh.f, h.weights, c[8]);
    if (!ok) return set_error(EFG_EIO, std::string("efg_load: ") + path + " is truncated");
    if (h.vlist[hd.n] != hd.m || h.offsets[hd.n] > h.data.size())
        return set_error(EFG_EIO, "efg_load: EFG arrays disagree with the header");
    h.n = hd.n;
    h.m = hd.m;
    h.m_input = hd.m_input;
    h.k = hd.k;
    h.row_lo = hd.row_lo;
    h.row_hi = hd.row_hi;
    h.symmetric = hd.symmetric != 0;
    h.fwd_bytes = hd.fwd_bytes;
    h.lower_bytes = hd.lower_bytes;
    h.upper_bytes = hd.upper_bytes;
    h.apriori_bits = hd.apriori_bits;
    h.build_seconds = 0.0;
    return EFG_OK;
}

}  // namespace efg
