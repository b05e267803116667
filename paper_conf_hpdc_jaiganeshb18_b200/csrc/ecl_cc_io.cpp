// ecl_cc_io.cpp — host-side graph readers beside the hot path.
//
// The paper's inputs came from the SuiteSparse/SMC collection (MatrixMarket files), SNAP
// (whitespace edge lists with '#' comments), DIMACS and Galois (§4).  These readers
// turn the two text formats into an undirected edge list in host memory; ecl_cc_build_csr
// then removes loops and multiple edges and adds back edges on the GPU, as the paper did.
// Plain C++ (one pass over the file in memory), no third-party code.
#include "ecl_cc.h"

#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

namespace {

thread_local char g_io_err[512] = {0};

ecl_cc_status io_fail(ecl_cc_status st, const char *fmt, ...)
{
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(g_io_err, sizeof(g_io_err), fmt, ap);
    va_end(ap);
    return st;
}

bool slurp(const char *path, std::string &buf)
{
    FILE *f = fopen(path, "rb");
    if (!f) return false;
    char tmp[1 << 16];
    size_t k;
    while ((k = fread(tmp, 1, sizeof(tmp), f)) > 0) buf.append(tmp, k);
    const bool ok = !ferror(f);
    fclose(f);
    return ok;
}

// cursor over the file text
struct Cur {
    const char *p, *e;
    long long line = 1;
    void skip_blank()
    {
        while (p < e && (*p == ' ' || *p == '\t' || *p == '\r')) p++;
    }
    bool eol() const { return p >= e || *p == '\n'; }
    void next_line()
    {
        while (p < e && *p != '\n') p++;
        if (p < e) {
            p++;
            line++;
        }
    }
    bool integer(long long &v)
    {
        skip_blank();
        bool neg = false;
        if (p < e && (*p == '-' || *p == '+')) neg = *p++ == '-';
        if (p >= e || *p < '0' || *p > '9') return false;
        long long x = 0;
        while (p < e && *p >= '0' && *p <= '9') {
            if (x > (1ll << 60)) return false;
            x = x * 10 + (*p++ - '0');
        }
        v = neg ? -x : x;
        return true;
    }
};

bool lower_eq(const char *a, size_t n, const char *b)
{
    if (strlen(b) != n) return false;
    for (size_t i = 0; i < n; i++)
        if ((a[i] | 0x20) != b[i]) return false;
    return true;
}

ecl_cc_status hand_out(std::vector<int32_t> &s, std::vector<int32_t> &d, int32_t n,
                       int32_t *n_out, int64_t *e_out, int32_t **src_out, int32_t **dst_out)
{
    const size_t E = s.size();
    int32_t *a = (int32_t *)malloc(sizeof(int32_t) * (E ? E : 1));
    int32_t *b = (int32_t *)malloc(sizeof(int32_t) * (E ? E : 1));
    if (!a || !b) {
        free(a);
        free(b);
        return io_fail(ECL_CC_ERR_OOM, "out of host memory");
    }
    if (E) {
        memcpy(a, s.data(), sizeof(int32_t) * E);
        memcpy(b, d.data(), sizeof(int32_t) * E);
    }
    *n_out = n;
    *e_out = (int64_t)E;
    *src_out = a;
    *dst_out = b;
    g_io_err[0] = 0;
    return ECL_CC_OK;
}

}  // namespace

extern "C" {

ecl_cc_status ecl_cc_read_mtx(const char *path, int32_t *n_out, int64_t *num_edges_out,
                              int32_t **src_out, int32_t **dst_out)
{
    if (!path || !n_out || !num_edges_out || !src_out || !dst_out)
        return io_fail(ECL_CC_ERR_INVALID_ARG, "null argument");
    std::string buf;
    if (!slurp(path, buf)) return io_fail(ECL_CC_ERR_INVALID_ARG, "cannot read %s", path);
    Cur c{buf.data(), buf.data() + buf.size()};
    // banner: %%MatrixMarket matrix coordinate <field> <symmetry>
    const char *b0 = c.p;
    while (!c.eol()) c.p++;
    std::vector<std::string> tok;
    for (const char *q = b0; q < c.p;) {
        while (q < c.p && (*q == ' ' || *q == '\t' || *q == '\r')) q++;
        const char *t = q;
        while (q < c.p && *q != ' ' && *q != '\t' && *q != '\r') q++;
        if (q > t) tok.emplace_back(t, q - t);
    }
    if (tok.size() < 5 || !lower_eq(tok[0].data(), tok[0].size(), "%%matrixmarket") ||
        !lower_eq(tok[1].data(), tok[1].size(), "matrix") ||
        !lower_eq(tok[2].data(), tok[2].size(), "coordinate"))
        return io_fail(ECL_CC_ERR_INVALID_GRAPH,
                       "%s: not a MatrixMarket coordinate file", path);
    int values = 0;   // numbers after "i j" on each entry line
    const std::string &fld = tok[3];
    if (lower_eq(fld.data(), fld.size(), "pattern")) values = 0;
    else if (lower_eq(fld.data(), fld.size(), "real") ||
             lower_eq(fld.data(), fld.size(), "integer") ||
             lower_eq(fld.data(), fld.size(), "double")) values = 1;
    else if (lower_eq(fld.data(), fld.size(), "complex")) values = 2;
    else return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: unknown field type", path);
    (void)values;   // values are ignored: an entry (i, j) is an edge whatever its weight
    c.next_line();
    while (c.p < c.e && (*c.p == '%' || *c.p == '\n' || *c.p == '\r')) c.next_line();
    long long rows = 0, cols = 0, nnz = 0;
    if (!c.integer(rows) || !c.integer(cols) || !c.integer(nnz) || rows < 0 || cols < 0 ||
        nnz < 0)
        return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: bad size line %lld", path, c.line);
    const long long nv = rows > cols ? rows : cols;
    if (nv > 0x7fffffffll) return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: too many vertices", path);
    c.next_line();
    std::vector<int32_t> s, d;
    s.reserve((size_t)nnz);
    d.reserve((size_t)nnz);
    for (long long k = 0; k < nnz; k++) {
        while (c.p < c.e && (*c.p == '%' || *c.p == '\n' || *c.p == '\r')) c.next_line();
        long long i = 0, j = 0;
        if (!c.integer(i) || !c.integer(j))
            return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: bad entry on line %lld", path, c.line);
        if (i < 1 || i > rows || j < 1 || j > cols)
            return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: index out of range on line %lld", path,
                           c.line);
        s.push_back((int32_t)(i - 1));
        d.push_back((int32_t)(j - 1));
        c.next_line();
    }
    return hand_out(s, d, (int32_t)nv, n_out, num_edges_out, src_out, dst_out);
}

ecl_cc_status ecl_cc_read_edgelist(const char *path, int32_t *n_out, int64_t *num_edges_out,
                                   int32_t **src_out, int32_t **dst_out)
{
    if (!path || !n_out || !num_edges_out || !src_out || !dst_out)
        return io_fail(ECL_CC_ERR_INVALID_ARG, "null argument");
    std::string buf;
    if (!slurp(path, buf)) return io_fail(ECL_CC_ERR_INVALID_ARG, "cannot read %s", path);
    Cur c{buf.data(), buf.data() + buf.size()};
    std::vector<int32_t> s, d;
    long long maxid = -1;
    while (c.p < c.e) {
        c.skip_blank();
        if (c.eol() || *c.p == '#' || *c.p == '%') {
            c.next_line();
            continue;
        }
        long long a = 0, b = 0;
        if (!c.integer(a) || !c.integer(b))
            return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: bad edge on line %lld", path, c.line);
        if (a < 0 || b < 0 || a > 0x7ffffffell || b > 0x7ffffffell)
            return io_fail(ECL_CC_ERR_INVALID_GRAPH, "%s: vertex ID out of range on line %lld",
                           path, c.line);
        s.push_back((int32_t)a);
        d.push_back((int32_t)b);
        if (a > maxid) maxid = a;
        if (b > maxid) maxid = b;
        c.next_line();
    }
    return hand_out(s, d, (int32_t)(maxid + 1), n_out, num_edges_out, src_out, dst_out);
}

void ecl_cc_free_host(void *p) { free(p); }

const char *ecl_cc_io_last_error(void) { return g_io_err; }

}  // extern "C"
